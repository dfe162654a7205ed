// capi.cu -- engine (buffer plan, step orchestration, CUDA graph) and the C
// ABI declared in include/nbody.h.  One time step = Alg. 6:
//   K1 bbox -> K2 keys -> K3 sort -> K4 permute -> K5 build -> K6 force -> K7 leapfrog
// all on the context stream, captured once into a CUDA graph and replayed.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>

#include <nvtx3/nvToolsExt.h>

#include "../../include/nbody.h"
#include "internal.cuh"

#ifdef NBODY_WITH_NCCL
#include <nccl.h>
#endif

using namespace nb;

struct nbody_ctx {
  int64_t n = 0;
  double theta = 0.5, eps = 0.0, dt = 0.0;
  int key_bits_opt = 16;
  int b = 16;
  int key_bytes = 8;
  bool use_graph = true;
  int traversal = 0;
  int build_variant = 0;  // 0 fused subtrees, 1 level by level
  bool timing = false;
  cudaEvent_t ev[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
  bool ev_valid = false;
  int kernels_per_step = 0;
  int device = 0;
  int nsm = kNumSMs;
  cudaStream_t stream = nullptr;
  cudaStream_t own_stream = nullptr;
  cudaStream_t cap_stream = nullptr;
  nbody_status state = NBODY_OK;
  std::string err;
  bool loaded = false;
  bool have_force = false;
  int64_t steps = 0;

  // device memory arena
  char* arena = nullptr;
  float4* pm[2] = {nullptr, nullptr};
  float4* vi[2] = {nullptr, nullptr};
  void* keys[2] = {nullptr, nullptr};
  uint32_t* idx[2] = {nullptr, nullptr};
  unsigned long long* keys_dbg = nullptr;
  float4* acc = nullptr;
  uint32_t* cnt = nullptr;
  float4* stage = nullptr;
  uint32_t* stage2 = nullptr;
  float* out3 = nullptr;
  float* bbox_part = nullptr;
  int nbbox = 0;
  GridInfo* grid = nullptr;
  unsigned long long* total = nullptr;
  int* bad = nullptr;
  SortPlan sort{};
  TreeView tree{};
  int perm_buf = 0;
  bool keys_dbg_valid = false;

  cudaGraph_t graph = nullptr;
  cudaGraphExec_t gexec = nullptr;
  cudaGraph_t graph_reuse = nullptr;    // tree-reuse step (NEXT-3(iii))
  cudaGraphExec_t gexec_reuse = nullptr;
  int sort_every = 1;                   // re-sort every k-th step
  bool last_sorted = false;
  void* quad_arena = nullptr;           // NEXT-4 S64 + qf (lazy)
  // caller-owned workspace (nbody_create_ws): every device buffer of the
  // context is carved from it in a fixed order; the library then allocates
  // no device memory of its own for the context's state
  bool ws_ext = false;
  char* ws = nullptr;
  size_t ws_bytes = 0, ws_used = 0;

  // partition over ranks [A21]: rank r owns sorted slots [own_b, own_e),
  // own_s = slice length (a multiple of 32 so warp groups match 1 GPU)
  int rank = 0, world = 1;
  int64_t own_s = 0, own_b = 0, own_e = 0;
#ifdef NBODY_WITH_NCCL
  ncclComm_t comm = nullptr;
  bool comm_borrowed = false;  // nbody_attach_comm: the caller's communicator, not destroyed here
#endif
  // fused K7 + exchange over peer memory (k_exchange.cu)
  size_t arena_bytes = 0;
  bool xpeer = false;
  PeerTable peers{};
  const float4* peer_acc[kMaxPeers] = {};
  const uint32_t* peer_cnt[kMaxPeers] = {};
  void* peer_map[kMaxPeers] = {};   // CUDA IPC mappings to close
  unsigned* xflags = nullptr;       // [kBarrierSlots][kMaxPeers] epochs signalled to this rank
  unsigned* xepoch = nullptr;       // [kBarrierSlots] this rank's barrier counters
  int* xerr = nullptr;              // set by a barrier that timed out
  // NEXT-2 FP64 mode
  bool f64 = false;
  void* arena64 = nullptr;
  double4* pm64[2] = {nullptr, nullptr};   // pm64[1] = the leaf ids of tree.rec64
  double4* vi64[2] = {nullptr, nullptr};
  double4* acc64 = nullptr;
  double* bbox_part64 = nullptr;
  double* stage64 = nullptr;               // [n][3] host-transfer staging
  // NEXT-3(i) cost-weighted ranges (peer exchange only)
  bool balance = false;
  uint32_t* gcost = nullptr;        // [ceil(n/32)] interactions per 32-slot group, last pass
  int64_t* dpart = nullptr;         // [kMaxPeers + 1] slot boundaries of the next pass
  int64_t* dpart_used = nullptr;    // [kMaxPeers + 1] boundaries of the last pass
  // K6a super-group lists (k_force.cu)
  uint32_t* sg_acc = nullptr;
  uint32_t* sg_fr = nullptr;
  int2* sg_cnt = nullptr;
  // pipelined host transfers (nbody_set_bodies_async / nbody_get_positions_async)
  cudaStream_t cstream = nullptr;   // copy stream, host -> device
  cudaStream_t ostream = nullptr;   // copy stream, device -> host (separate: it waits for steps)
  char* xfer = nullptr;             // in_stage[2] (28 B/body) + out_stage[2] (12 B/body)
  int* bad_async = nullptr;         // validation flags of async input sets since the last sync
  cudaEvent_t ev_in_copied[2] = {}, ev_in_used[2] = {}, ev_out_ready[2] = {}, ev_out_copied[2] = {};
  bool ev_in_used_rec[2] = {}, ev_out_copied_rec[2] = {};
  int slot_in = 0, slot_out = 0;
};

namespace {

const char* status_name(nbody_status s) {
  switch (s) {
    case NBODY_OK: return "ok";
    case NBODY_EINVAL: return "invalid argument";
    case NBODY_ENOMEM: return "out of device memory";
    case NBODY_ECUDA: return "CUDA error";
    case NBODY_ENCCL: return "NCCL error";
    case NBODY_ESTATE: return "bad state";
  }
  return "?";
}

nbody_status fail(nbody_ctx* c, nbody_status s, const std::string& msg) {
  if (c) {
    c->err = std::string(status_name(s)) + ": " + msg;
    if (s == NBODY_ECUDA || s == NBODY_ENCCL) c->state = NBODY_ESTATE;
  }
  return s;
}

#define CK(call)                                                                              \
  do {                                                                                        \
    cudaError_t e_ = (call);                                                                  \
    if (e_ != cudaSuccess) return fail(c, NBODY_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

#define CHECK_CTX(c)                                             \
  do {                                                           \
    if (!(c)) return NBODY_EINVAL;                               \
    if ((c)->state != NBODY_OK) return NBODY_ESTATE;             \
  } while (0)

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

int resolve_bits(int64_t n, int opt) {
  if (opt > 0) return opt;
  int b = 1;
  while (b < 21 && (uint64_t(1) << (3 * b)) < uint64_t(n)) ++b;  // [A8] smallest b with 8^b >= N
  return b;
}

size_t align_up(size_t x) { return (x + 255) & ~size_t(255); }

constexpr int kMaxWorld = 256;
constexpr int64_t kPartPad = 256 * kMaxWorld;  // G * S - N < 256 G

// [A21] S = ceil(N / G) rounded up to a multiple of kPartUnit = 256 slots:
// the warp groups (32) and K6a's super-groups (kSG = 256) then coincide
// with the single-GPU run, so results are bit-identical.
constexpr int64_t kPartUnit = kPartUnitSlots;
static_assert(kSG <= 0 || kPartUnit % kSG == 0, "rank ranges must start at super-group boundaries");
void set_part(nbody_ctx* c, int rank, int world) {
  const int64_t n = c->n;
  int64_t s = (n + world - 1) / world;
  s = (s + kPartUnit - 1) / kPartUnit * kPartUnit;
  c->rank = rank;
  c->world = world;
  c->own_s = s;
  c->own_b = std::min(n, int64_t(rank) * s);
  c->own_e = std::min(n, int64_t(rank + 1) * s);
}

// Tree plan (sizes follow from N alone).  Heap numbering: node
// (l, j) has global id g = 2^(L-l) + j, so the root is 1, the children of g
// are 2g and 2g+1 and leaf i is 2^L + i; level l only uses its first
// ceil(N / 2^l) ids.  Returns the number of ids (2^(L+1)).
int64_t plan_tree(TreeView& t, int64_t n) {
  t.n = n;
  t.L = 0;
  while ((int64_t(1) << t.L) < n) ++t.L;
  t.count[0] = n;
  t.off[0] = int64_t(1) << t.L;
  for (int l = 1; l <= t.L; ++l) {
    t.count[l] = (t.count[l - 1] + 1) / 2;
    t.off[l] = int64_t(1) << (t.L - l);
  }
  for (int l = t.L + 1; l < kMaxLevels; ++l) t.count[l] = t.off[l] = 0;
  return int64_t(2) << t.L;
}

// Sizes of the base arena's buffers, in carving order (sz[32]); returns the
// count.  Depends on N (tree sizes are fixed by N) and the SM count
// (bbox partials) only: every key width (b <= 21) and every world <= 256
// fit the same layout.
int arena_plan(int64_t n, int nsm, size_t* sz) {
  TreeView t{};
  const int64_t ids = plan_tree(t, n);         // rec / s2f cover leaves too
  const int64_t inner = ids / 2;                // pred / mom / box: internal ids < 2^L
  const int nbbox = 2 * nsm;
  const int64_t tiles = sort_tiles(n);
  int k = 0;
  sz[k++] = 16 * size_t(n + kPartPad);              // pm0 (room for G * S records)
  sz[k++] = 16 * size_t(n + kPartPad);              // vi0
  sz[k++] = 16 * size_t(n);                         // vi1
  sz[k++] = 8 * size_t(n);                          // keys0
  sz[k++] = 8 * size_t(n);                          // keys1
  sz[k++] = 4 * size_t(n);                          // idx0
  sz[k++] = 4 * size_t(n);                          // idx1
  sz[k++] = 8 * size_t(n);                          // keys_dbg
  sz[k++] = 16 * size_t(n);                         // acc
  sz[k++] = 4 * size_t(n);                          // cnt
  sz[k++] = 16 * size_t(n + kPartPad);              // stage (gathered acc for G > 1)
  sz[k++] = 4 * size_t(n + kPartPad);               // stage2 (gathered counts)
  sz[k++] = 12 * size_t(n);                         // out3 (by-id outputs for host callers)
  sz[k++] = sizeof(float) * 6 * size_t(nbbox);   // bbox partials
  sz[k++] = sizeof(GridInfo);
  sz[k++] = 8;                                      // total
  sz[k++] = 8;                                      // bad
  sz[k++] = sort_scratch_bytes(n);                  // sort
  sz[k++] = 32 * size_t(inner);                     // pred
  sz[k++] = 16 * size_t(ids);                       // rec (leaf ids hold the sorted bodies)
  sz[k++] = 32 * size_t(inner);                     // mom
  sz[k++] = 16 * size_t(inner);                     // blo
  sz[k++] = 16 * size_t(inner);                     // bhi
  sz[k++] = 8 * size_t(ids);                        // rc (-inf at the leaves)
  sz[k++] = 16 * size_t(inner);                     // tf
  sz[k++] = 4 * size_t(n / 32 + 1);                 // gcost
  sz[k++] = 512;                                    // exchange flags, epochs, error, partitions
  sz[k++] = 4 * size_t(kSGAcc) * size_t(sg_groups(n));  // K6a super-group lists: accepted
  sz[k++] = 4 * size_t(kSGFr) * size_t(sg_groups(n));   //   frontier
  sz[k++] = 8 * size_t(sg_groups(n)) + 8;               //   counts
  return k;
}

size_t sum_aligned(const size_t* sz, int k) {
  size_t total = 0;
  for (int i = 0; i < k; ++i) total += align_up(sz[i]);
  return total;
}

size_t arena_bytes_for(int64_t n, int nsm) {
  size_t sz[32];
  return sum_aligned(sz, arena_plan(n, nsm, sz));
}

// Optional buffers, allocated on first use (NBODY_WS_* in nbody.h).
size_t quad_bytes_for(int64_t n) {
  TreeView t{};
  const size_t inner = size_t(plan_tree(t, n) / 2);
  return align_up(48 * inner + 32 * inner);
}
size_t xfer_bytes_for(int64_t n) { return align_up(align_up(2 * 28 * size_t(n)) + align_up(2 * 12 * size_t(n)) + 256); }
size_t f64_plan(int64_t n, int nsm, size_t* sz) {
  TreeView t{};
  const size_t ids = size_t(plan_tree(t, n)), inner = ids / 2;
  const int nbbox = 2 * nsm;
  int k = 0;
  sz[k++] = 32 * size_t(n);              // pm64[0]
  sz[k++] = 32 * size_t(n);              // vi64[0]
  sz[k++] = 32 * size_t(n);              // vi64[1]
  sz[k++] = 32 * ids;                    // rec64 (leaf ids = pm64[1])
  sz[k++] = 32 * inner;                  // blo64
  sz[k++] = 32 * inner;                  // bhi64
  sz[k++] = 32 * size_t(n);              // acc64
  sz[k++] = 48 * size_t(nbbox) + 24 * size_t(n);  // bbox partials + staging
  return size_t(k);
}
size_t f64_bytes_for(int64_t n, int nsm) {
  size_t sz[8];
  return sum_aligned(sz, int(f64_plan(n, nsm, sz)));
}

// Device memory for the context: from the caller's workspace (create_ws),
// else cudaMalloc.  `what` names the buffer in the error.
// The memory is zeroed once: some kernels load whole sibling pairs or
// vectors that include never-written slots (the missing right sibling at the
// ragged end of a level) and discard them; zero-filled, those reads are of
// defined memory (compute-sanitizer initcheck is clean).
nbody_status dev_alloc(nbody_ctx* c, size_t bytes, void** out, const char* what) {
  *out = nullptr;
  bytes = align_up(bytes);
  if (c->ws_ext) {
    if (c->ws_used + bytes > c->ws_bytes)
      return fail(c, NBODY_ENOMEM, std::string(what) + ": the caller's workspace is too small (" +
                                       std::to_string(c->ws_bytes) + " bytes; nbody_workspace_bytes_ex gives the size "
                                       "with the optional buffers)");
    *out = c->ws + c->ws_used;
    c->ws_used += bytes;
  } else {
    const cudaError_t e = cudaMalloc(out, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      *out = nullptr;
      return fail(c, NBODY_ENOMEM, std::string(what) + ": cudaMalloc of " + std::to_string(bytes) + " bytes failed");
    }
  }
  CK(cudaMemsetAsync(*out, 0, bytes, c->stream ? c->stream : cudaStreamLegacy));
  CK(cudaStreamSynchronize(c->stream ? c->stream : cudaStreamLegacy));
  return NBODY_OK;
}
void dev_free(nbody_ctx* c, void* p) {
  if (p && !c->ws_ext) cudaFree(p);
}

nbody_status allocate(nbody_ctx* c) {
  const int64_t n = c->n;
  plan_tree(c->tree, n);
  c->nbbox = 2 * c->nsm;
  const int64_t tiles = sort_tiles(n);
  size_t sz[32];
  const int k = arena_plan(n, c->nsm, sz);
  const size_t total = sum_aligned(sz, k);
  {
    void* a = nullptr;
    const nbody_status st = dev_alloc(c, total, &a, "state and tree arena");
    if (st != NBODY_OK) return st;
    c->arena = static_cast<char*>(a);
  }
  char* p = c->arena;
  int i = 0;
  auto take = [&](void) -> char* { char* r = p; p += align_up(sz[i++]); return r; };
  c->pm[0] = (float4*)take();
  c->vi[0] = (float4*)take();
  c->vi[1] = (float4*)take();
  c->keys[0] = take();
  c->keys[1] = take();
  c->idx[0] = (uint32_t*)take();
  c->idx[1] = (uint32_t*)take();
  c->keys_dbg = (unsigned long long*)take();
  c->acc = (float4*)take();
  c->cnt = (uint32_t*)take();
  c->stage = (float4*)take();
  c->stage2 = (uint32_t*)take();
  c->out3 = (float*)take();
  c->bbox_part = (float*)take();
  c->grid = (GridInfo*)take();
  c->total = (unsigned long long*)take();
  c->bad = (int*)take();
  char* sortmem = take();
  c->tree.pred = (double4*)take();
  c->tree.rec = (float4*)take();
  c->tree.mom = (double4*)take();
  c->tree.blo = (float4*)take();
  c->tree.bhi = (float4*)take();
  c->tree.rc = (float2*)take();
  c->tree.tf = (float4*)take();
  c->gcost = (uint32_t*)take();
  c->xflags = (unsigned*)take();
  c->xepoch = c->xflags + kBarrierSlots * kMaxPeers;
  c->xerr = reinterpret_cast<int*>(c->xepoch + kBarrierSlots);
  c->sg_acc = (uint32_t*)take();
  c->sg_fr = (uint32_t*)take();
  c->sg_cnt = (int2*)take();
  c->dpart = reinterpret_cast<int64_t*>(reinterpret_cast<char*>(c->xflags) + 128);
  c->dpart_used = c->dpart + kMaxPeers + 1;
  c->arena_bytes = total;
  c->tree.grid = c->grid;
  c->tree.th2 = c->theta * c->theta;
  // the sorted bodies live in the leaf ids of the record array
  c->pm[1] = c->tree.rec + (int64_t(1) << c->tree.L);
  // leaves always interact when reached: thresholds (-inf, -inf), set once
  const float ninf = -INFINITY;
  launch_fill_float2(c->tree.rc + (int64_t(1) << c->tree.L), n, make_float2(ninf, ninf), nullptr);
  cudaError_t e = cudaMemset(c->xflags, 0, 512);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return fail(c, NBODY_ECUDA, cudaGetErrorString(e));
  c->sort.n = n;
  c->sort.tiles = tiles;
  c->sort.ghist = (uint32_t*)sortmem;
  c->sort.tile_ctr = c->sort.ghist + 8 * 256;
  c->sort.gpre = c->sort.tile_ctr + 8;
  c->sort.status = c->sort.gpre + 8 * 256;
  return NBODY_OK;
}

// NEXT-2 FP64 mode buffers (one allocation, on first use).
nbody_status alloc_f64(nbody_ctx* c) {
  const int64_t n = c->n;
  size_t sz[8];
  f64_plan(n, c->nsm, sz);
  {
    const nbody_status st = dev_alloc(c, sum_aligned(sz, 8), &c->arena64, "FP64 mode buffers");
    if (st != NBODY_OK) return st;
  }
  char* p = static_cast<char*>(c->arena64);
  int i = 0;
  auto take = [&](void) -> char* { char* r = p; p += align_up(sz[i++]); return r; };
  c->pm64[0] = (double4*)take();
  c->vi64[0] = (double4*)take();
  c->vi64[1] = (double4*)take();
  double4* rec64 = (double4*)take();
  c->pm64[1] = rec64 + (int64_t(1) << c->tree.L);
  c->tree.blo64 = (double4*)take();
  c->tree.bhi64 = (double4*)take();
  c->acc64 = (double4*)take();
  c->bbox_part64 = (double*)take();
  c->stage64 = c->bbox_part64 + 6 * size_t(c->nbbox);
  return NBODY_OK;
}

// S1 fused into K7: valid when one rank updates every body
// (fp32 mode); the bbox partials are then always those of the current
// state: set_bodies* computes them after packing, K7 after updating, and a
// force-only pass only permutes the bodies (min/max of the same set).
bool bbox_fused(const nbody_ctx* c) {
  bool comm = false;
#ifdef NBODY_WITH_NCCL
  comm = c->comm != nullptr;
#endif
  return !c->f64 && c->world == 1 && !c->xpeer && !comm;
}

// NEXT-3(i) is active: peer exchange over G > 1 ranks with balance on.
bool balanced(const nbody_ctx* c) { return c->balance && c->xpeer && c->world > 1; }

// Rank q's slot range in the last force pass (host view; syncs when the
// ranges live on the device).
nbody_status rank_range(nbody_ctx* c, int q, int64_t* b, int64_t* e) {
  if (!balanced(c)) return nbody_partition(c->n, q, c->world, b, e);
  int64_t r[2];
  CK(cudaMemcpyAsync(r, c->dpart_used + q, sizeof(r), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  *b = r[0];
  *e = r[1];
  return NBODY_OK;
}

void drop_graph(nbody_ctx* c) {
  if (c->gexec) cudaGraphExecDestroy(c->gexec);
  if (c->graph) cudaGraphDestroy(c->graph);
  if (c->gexec_reuse) cudaGraphExecDestroy(c->gexec_reuse);
  if (c->graph_reuse) cudaGraphDestroy(c->graph_reuse);
  c->gexec = nullptr;
  c->graph = nullptr;
  c->gexec_reuse = nullptr;
  c->graph_reuse = nullptr;
}

// One force pass (and optionally the update) on stream s.  State enters in
// (pm[0], vi[0]) in the current slot order and leaves there in the new
// Hilbert order.
nbody_status enqueue_pass(nbody_ctx* c, cudaStream_t s, bool integrate, bool debug, bool resort = true) {
  const int64_t n = c->n;
  const bool tm = c->timing && s == c->stream;
  // stage boundaries: CUDA events (NBODY_OPT_TIMING, graphs off) and NVTX
  // ranges around each stage's enqueue (the paper's per-component times,
  // P:298; host-side, so they bracket the launches with graphs off and
  // the capture with graphs on)
  static const char* const kStage[5] = {"S1-S2 bbox + Hilbert keys", "S3 radix sort", "S4-S5 permute + build",
                                        "S6 force (K6a + K6)", "S7 update (+ exchange)"};
  auto mark = [&](int i) -> cudaError_t {
    if (i > 0) nvtxRangePop();
    if (i < 5) nvtxRangePushA(kStage[i]);
    return tm ? cudaEventRecord(c->ev[i], s) : cudaSuccess;
  };
  CK(mark(0));
  const bool f64 = c->f64;
  if (f64) {  // NEXT-2: fp64 bodies
    launch_bbox_partial_f64(c->pm64[0], n, c->bbox_part64, c->nbbox, s);
    launch_bbox_final_f64(c->bbox_part64, c->nbbox, c->b, c->grid, s);
  } else {
    // S1: the partials come from the previous K7 (or the packing of
    // set_bodies) on one rank; ranks that update a slice re-read all bodies
    if (!bbox_fused(c)) launch_bbox_partial(c->pm[0], n, c->bbox_part, c->nbbox, s);
    launch_bbox_final(c->bbox_part, c->nbbox, c->b, c->grid, s);
  }
  int front_kernels = f64 || !bbox_fused(c) ? 2 : 1;
  if (resort) {
    CK(cudaMemsetAsync(c->sort.ghist, 0, sizeof(uint32_t) * 8 * 256, s));
    c->sort.hist_ready = true;  // the key kernel fills the sort's digit histograms
    if (f64)
      launch_keys_f64(c->pm64[0], n, c->grid, c->keys[0], c->key_bytes, c->sort.ghist, c->sort.passes, s);
    else if (c->key_bytes == 4)
      launch_keys32(c->pm[0], n, c->grid, static_cast<uint32_t*>(c->keys[0]), c->sort.ghist, c->sort.passes, s);
    else
      launch_keys64(c->pm[0], n, c->grid, static_cast<unsigned long long*>(c->keys[0]), c->sort.ghist,
                    c->sort.passes, c->b, s);
    if (debug) {
      CK(cudaMemcpyAsync(c->keys_dbg, c->keys[0], size_t(c->key_bytes) * n, cudaMemcpyDeviceToDevice, s));
    }
    CK(mark(1));
    c->perm_buf = launch_radix_sort(c->sort, c->keys, c->idx, s);
    CK(mark(2));
    if (f64)
      launch_permute_f64(c->pm64[0], c->vi64[0], c->idx[c->perm_buf], n, c->pm64[1], c->vi64[1], s);
    else
      launch_permute(c->pm[0], c->vi[0], c->idx[c->perm_buf], n, c->pm[1], c->vi[1], s);
    front_kernels += 1 + 1 + c->sort.passes + 1;  // keys, digit prefix, sort passes, permute
  } else {
    // tree reuse (NEXT-3(iii), [A23]): keep the current (previous Hilbert)
    // order; the leaves are the current state
    CK(mark(1));
    CK(mark(2));
    if (f64) {
      CK(cudaMemcpyAsync(c->pm64[1], c->pm64[0], 32 * size_t(n), cudaMemcpyDeviceToDevice, s));
      CK(cudaMemcpyAsync(c->vi64[1], c->vi64[0], 32 * size_t(n), cudaMemcpyDeviceToDevice, s));
    } else {
      CK(cudaMemcpyAsync(c->pm[1], c->pm[0], 16 * size_t(n), cudaMemcpyDeviceToDevice, s));
      CK(cudaMemcpyAsync(c->vi[1], c->vi[0], 16 * size_t(n), cudaMemcpyDeviceToDevice, s));
    }
  }
  c->last_sorted = resort;
  int x_kernels = 0;
  if (c->xpeer) {  // every rank has consumed the old state: peers may overwrite it (and, for a
                   // force-only pass, no peer still reads the acc/cnt/gcost this pass rewrites)
    launch_xbarrier(c->peers, c->xepoch, 0, c->xerr, s);
    ++x_kernels;
  }
  int build_kernels;
  if (f64) {  // NEXT-2: fp64 leaves at tree.rec64 + 2^L, fp64 boxes
    launch_build_fused_f64(c->tree, debug, s);
    build_kernels = c->tree.L < 1 ? 0 : (c->tree.L > 9 ? 2 : 1);
  } else if (c->build_variant == 1 && !c->tree.quad) {  // the level-by-level variant is monopole only
    launch_build(c->tree, c->pm[1], s);
    build_kernels = c->tree.L;
  } else {
    launch_build_fused(c->tree, c->pm[1], debug, s);
    build_kernels = build_fused_kernels(c->tree);
  }
  CK(cudaMemsetAsync(c->total, 0, sizeof(unsigned long long), s));
  CK(mark(3));
  // S6/S7 only on the owned sorted slots [own_b, own_e) [A21]
  const int64_t ob = c->own_b, oe = c->own_e;
  ForceParams fp;
  fp.t = c->tree;
  fp.leaves = c->pm[1];
  fp.grid = c->grid;
  fp.t_begin = ob;
  fp.t_end = oe;
  fp.th2 = c->theta * c->theta;
  fp.eps2 = float(c->eps * c->eps);
  fp.acc = c->acc;
  fp.count = c->cnt;
  fp.total = c->total;
  if (f64) {  // NEXT-2 (tree.rec64 is set: K6 runs its fp64 variant)
    fp.leaves64 = c->pm64[1];
    fp.acc64 = c->acc64;
    fp.eps2_64 = c->eps * c->eps;
  }
  const bool bal = balanced(c);
  const int64_t groups = (n + 31) / 32;                      // 32-slot cost groups (one per K6 warp)
  const int64_t units = (n + kPartUnit - 1) / kPartUnit;      // 256-slot partition units [A21]
  const int64_t cap_units = std::min(units, 2 * ((units + c->world - 1) / c->world));
  if (bal) {  // NEXT-3(i): the range is read on the device
    fp.part = c->dpart;
    fp.part_rank = c->rank;
    fp.cap = std::min(n, kPartUnit * cap_units);
    fp.xp = c->peers;
  }
  int sg_kernels = 0;
  if (c->traversal == 0 && kSG > 0) {  // K6a, then K6 continues from its lists
    fp.sg_acc = c->sg_acc;
    fp.sg_fr = c->sg_fr;
    fp.sg_cnt = c->sg_cnt;
    launch_force_sgroups(fp, s);
    sg_kernels = 1;
  }
  launch_force(fp, c->traversal, s);
  CK(mark(4));
  if (integrate && c->xpeer) {
    // K7 stores the owned records into every rank's state, then the
    // delivery barrier (k_exchange.cu)
    launch_leapfrog_scatter(c->pm[1], c->vi[1], c->acc, ob, bal ? fp.cap : oe - ob, float(c->dt), c->peers,
                            bal ? c->dpart : nullptr, s);
    launch_xbarrier(c->peers, c->xepoch, 1, c->xerr, s);
    ++x_kernels;
    if (bal) {  // every group cost has landed: next pass's ranges
      launch_partition(c->gcost, groups, c->world, n, cap_units, c->dpart, c->dpart_used, s);
      ++x_kernels;
    }
  } else if (integrate && f64) {
    launch_leapfrog_f64(c->pm64[1] + ob, c->vi64[1] + ob, c->acc64, oe - ob, c->dt, c->pm64[0] + ob,
                        c->vi64[0] + ob, s);
  } else if (integrate && bbox_fused(c)) {  // K7 + the next pass's S1 partials (one rank, all bodies)
    launch_leapfrog_bbox(c->pm[1], c->vi[1], c->acc, n, float(c->dt), c->pm[0], c->vi[0], c->bbox_part, c->nbbox, s);
  } else if (integrate) {
    launch_leapfrog(c->pm[1] + ob, c->vi[1] + ob, c->acc, oe - ob, float(c->dt), c->pm[0] + ob, c->vi[0] + ob, s);
#ifdef NBODY_WITH_NCCL
    if (c->comm) {  // S0 of the next step: every rank gets every owned slice
      const size_t cnt = 4 * size_t(c->own_s);
      ncclResult_t r = ncclGroupStart();
      if (r == ncclSuccess)
        r = ncclAllGather(c->pm[0] + int64_t(c->rank) * c->own_s, c->pm[0], cnt, ncclFloat, c->comm, s);
      if (r == ncclSuccess)
        r = ncclAllGather(c->vi[0] + int64_t(c->rank) * c->own_s, c->vi[0], cnt, ncclFloat, c->comm, s);
      const ncclResult_t r2 = ncclGroupEnd();
      if (r != ncclSuccess || r2 != ncclSuccess)
        return fail(c, NBODY_ENCCL, ncclGetErrorString(r != ncclSuccess ? r : r2));
    }
#endif
  } else if (f64) {
    CK(cudaMemcpyAsync(c->pm64[0], c->pm64[1], 32 * size_t(n), cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(c->vi64[0], c->vi64[1], 32 * size_t(n), cudaMemcpyDeviceToDevice, s));
  } else {
    CK(cudaMemcpyAsync(c->pm[0], c->pm[1], 16 * size_t(n), cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(c->vi[0], c->vi[1], 16 * size_t(n), cudaMemcpyDeviceToDevice, s));
    if (c->xpeer) {  // every rank's forces are final before a getter reads them
      launch_xbarrier(c->peers, c->xepoch, 1, c->xerr, s);
      ++x_kernels;
      if (bal) {
        launch_partition(c->gcost, groups, c->world, n, cap_units, c->dpart, c->dpart_used, s);
        ++x_kernels;
      }
    }
  }
  CK(mark(5));
  c->ev_valid = tm;
  // K1 2 + K2 (with the digit histograms) 1 + K3 passes + K4 1 + K5 + K6 1 + K7 1
  c->kernels_per_step = front_kernels + build_kernels + 1 + sg_kernels + (integrate ? 1 : 0) + x_kernels;
  CK(cudaGetLastError());
  return NBODY_OK;
}

// Capture one full step (resort = sorting step, else tree-reuse step).
nbody_status build_graph(nbody_ctx* c, bool resort) {
  cudaGraph_t& graph = resort ? c->graph : c->graph_reuse;
  cudaGraphExec_t& exec = resort ? c->gexec : c->gexec_reuse;
  CK(cudaStreamBeginCapture(c->cap_stream, cudaStreamCaptureModeThreadLocal));
  nbody_status st = enqueue_pass(c, c->cap_stream, true, false, resort);
  cudaGraph_t g = nullptr;
  cudaError_t e = cudaStreamEndCapture(c->cap_stream, &g);
  if (st != NBODY_OK) {
    if (g) cudaGraphDestroy(g);
    return st;
  }
  if (e != cudaSuccess) return fail(c, NBODY_ECUDA, std::string("graph capture: ") + cudaGetErrorString(e));
  graph = g;
  CK(cudaGraphInstantiate(&exec, g, 0));
  return NBODY_OK;
}

nbody_status sync_stream(nbody_ctx* c) {
  CK(cudaStreamSynchronize(c->stream));
  if (c->xpeer) {
    int err = 0;
    CK(cudaMemcpyAsync(&err, c->xerr, sizeof(int), cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    if (err) {
      c->state = NBODY_ESTATE;
      c->err = "peer exchange: a barrier timed out (a rank stopped stepping); the state is invalid";
      return NBODY_ESTATE;
    }
  }
  return NBODY_OK;
}

// Fill the peer table from every rank's arena base (layouts are identical:
// same N, same plan) and switch the context to the fused exchange.
nbody_status attach_peer_bases(nbody_ctx* c, char* const* base, int rank, int world) {
  auto at = [&](int q, const void* own) { return base[q] + (static_cast<const char*>(own) - c->arena); };
  PeerTable& pt = c->peers;
  pt.G = world;
  pt.rank = rank;
  for (int q = 0; q < world; ++q) {
    pt.pm[q] = (float4*)at(q, c->pm[0]);
    pt.vi[q] = (float4*)at(q, c->vi[0]);
    pt.flags[q] = (unsigned*)at(q, c->xflags);
    pt.gcost[q] = (uint32_t*)at(q, c->gcost);
    c->peer_acc[q] = (const float4*)at(q, c->acc);
    c->peer_cnt[q] = (const uint32_t*)at(q, c->cnt);
  }
  set_part(c, rank, world);
  c->xpeer = true;
  // NEXT-3(i): the first pass uses the equal slices [A21]
  int64_t bounds[kMaxPeers + 1];
  for (int q = 0; q <= world; ++q) bounds[q] = std::min(c->n, int64_t(q) * c->own_s);
  CK(cudaMemcpyAsync(c->dpart, bounds, sizeof(int64_t) * (world + 1), cudaMemcpyHostToDevice, c->stream));
  CK(cudaMemcpyAsync(c->dpart_used, bounds, sizeof(int64_t) * (world + 1), cudaMemcpyHostToDevice, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  drop_graph(c);
  return NBODY_OK;
}

struct PeerDesc {  // nbody_peer_handle's 128-byte record
  cudaIpcMemHandle_t ipc;
  int64_t n;
  uint64_t arena_bytes;
  uint32_t magic;
  char pci[20];     // the owner's device, as a PCI bus id (device ordinals differ between processes)
  uint64_t offset;  // the arena's offset in the allocation the IPC handle maps (a caller workspace,
                    // e.g. a torch tensor, may sit inside a larger cudaMalloc block)
};

// Base address of the device allocation containing p (driver API
// cuMemGetAddressRange, reached through the runtime's entry-point query so
// the library needs no libcuda link).
nbody_status alloc_base(nbody_ctx* c, const void* p, const char** base) {
  using Fn = int (*)(unsigned long long*, size_t*, unsigned long long);
  static Fn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion("cuMemGetAddressRange", &f, 12000, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !f) {
      cudaGetLastError();
      return fail(c, NBODY_ECUDA, "cuMemGetAddressRange is not available");
    }
    fn = reinterpret_cast<Fn>(f);
  }
  unsigned long long b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, reinterpret_cast<unsigned long long>(p)) != 0)
    return fail(c, NBODY_ECUDA, "cuMemGetAddressRange failed for the arena");
  *base = reinterpret_cast<const char*>(b);
  return NBODY_OK;
}
static_assert(sizeof(PeerDesc) <= 128, "peer descriptor must fit in 128 bytes");
constexpr uint32_t kPeerMagic = 0x4e42584bu;

}  // namespace

extern "C" {

int nbody_version(void) { return 100; }

nbody_status nbody_select_device(int device) {
  int count = 0;
  if (cudaGetDeviceCount(&count) != cudaSuccess) {
    cudaGetLastError();
    return NBODY_ECUDA;
  }
  if (device < 0 || device >= count) return NBODY_EINVAL;
  return cudaSetDevice(device) == cudaSuccess ? NBODY_OK : NBODY_ECUDA;
}

static void preload_all() {
  static bool done = false;  // per process; kernels are loaded per context, and the library uses one device context
  if (done) return;
  done = true;
  preload_allpairs();
  preload_bbox_keys();
  preload_build();
  preload_direct();
  preload_exchange();
  preload_force();
  preload_update();
  preload_sort();
}

static nbody_status create_impl(int64_t n, double theta, double eps, double dt, void* ws, size_t ws_bytes,
                                nbody_ctx** out) {
  if (!out) return NBODY_EINVAL;
  *out = nullptr;
  if (n < 1 || n >= (int64_t(1) << 30)) return NBODY_EINVAL;
  if (!std::isfinite(theta) || theta < 0 || !std::isfinite(eps) || eps < 0 || !std::isfinite(dt)) return NBODY_EINVAL;
  if (ws && (reinterpret_cast<uintptr_t>(ws) & 255u)) return NBODY_EINVAL;  // 256-byte aligned (torch: 512)
  nbody_ctx* c = new (std::nothrow) nbody_ctx;
  if (!c) return NBODY_ENOMEM;
  c->n = n;
  c->theta = theta;
  c->eps = eps;
  c->dt = dt;
  auto bail = [&](nbody_status s) {
    nbody_destroy(c);
    return s;
  };
  if (cudaGetDevice(&c->device) != cudaSuccess) return bail(NBODY_ECUDA);
  cudaDeviceGetAttribute(&c->nsm, cudaDevAttrMultiProcessorCount, c->device);
  if (c->nsm <= 0) c->nsm = kNumSMs;
  if (ws) {
    if (!is_device_ptr(ws)) return bail(NBODY_EINVAL);
    cudaPointerAttributes pa;
    if (cudaPointerGetAttributes(&pa, ws) != cudaSuccess || pa.device != c->device) {
      cudaGetLastError();
      return bail(NBODY_EINVAL);  // the workspace must live on the current device
    }
    if (ws_bytes < arena_bytes_for(n, c->nsm)) return bail(NBODY_ENOMEM);
    c->ws_ext = true;
    c->ws = static_cast<char*>(ws);
    c->ws_bytes = ws_bytes;
  }
  if (cudaStreamCreateWithFlags(&c->own_stream, cudaStreamNonBlocking) != cudaSuccess) return bail(NBODY_ECUDA);
  if (cudaStreamCreateWithFlags(&c->cap_stream, cudaStreamNonBlocking) != cudaSuccess) return bail(NBODY_ECUDA);
  for (auto& e : c->ev)
    if (cudaEventCreate(&e) != cudaSuccess) return bail(NBODY_ECUDA);
  c->stream = c->own_stream;
  preload_all();
  nbody_status s = allocate(c);
  if (s != NBODY_OK) return bail(s);
  set_part(c, 0, 1);
  c->b = resolve_bits(n, c->key_bits_opt);
  c->key_bytes = 3 * c->b <= 32 ? 4 : 8;
  c->sort.key_bytes = c->key_bytes;
  c->sort.passes = (3 * c->b + 7) / 8;
  *out = c;
  return NBODY_OK;
}

nbody_status nbody_create(int64_t n, double theta, double eps, double dt, nbody_ctx** out) {
  return create_impl(n, theta, eps, dt, nullptr, 0, out);
}

nbody_status nbody_create_ws(int64_t n, double theta, double eps, double dt, void* dev_workspace, size_t bytes,
                             nbody_ctx** out) {
  if (!dev_workspace) {
    if (out) *out = nullptr;
    return NBODY_EINVAL;
  }
  return create_impl(n, theta, eps, dt, dev_workspace, bytes, out);
}

static int current_sms() {
  int dev = 0, nsm = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
    cudaGetLastError();
    nsm = kNumSMs;
  }
  return nsm > 0 ? nsm : kNumSMs;
}

size_t nbody_workspace_bytes_ex(int64_t n, int world, int key_bits, unsigned features) {
  if (n < 1 || n >= (int64_t(1) << 30) || world < 1 || world > kMaxWorld || key_bits < 0 || key_bits > 21) return 0;
  if (features & ~unsigned(NBODY_WS_QUAD | NBODY_WS_XFER | NBODY_WS_FP64)) return 0;
  const int nsm = current_sms();
  size_t total = arena_bytes_for(n, nsm);  // one layout for every world <= 256 and b <= 21
  if (features & NBODY_WS_QUAD) total += quad_bytes_for(n);
  if (features & NBODY_WS_XFER) total += xfer_bytes_for(n);
  if (features & NBODY_WS_FP64) total += align_up(f64_bytes_for(n, nsm));
  return total;
}

size_t nbody_workspace_bytes(int64_t n, int world, int key_bits) {
  return nbody_workspace_bytes_ex(n, world, key_bits, 0u);
}

nbody_status nbody_set_option(nbody_ctx* c, int option, int64_t value) {
  CHECK_CTX(c);
  switch (option) {
    case NBODY_OPT_KEY_BITS:
      if (value < 0 || value > 21) return fail(c, NBODY_EINVAL, "key bits must be in [0, 21]");
      c->key_bits_opt = int(value);
      c->b = resolve_bits(c->n, c->key_bits_opt);
      c->key_bytes = 3 * c->b <= 32 ? 4 : 8;
      c->sort.key_bytes = c->key_bytes;
      c->sort.passes = (3 * c->b + 7) / 8;
      drop_graph(c);
      return NBODY_OK;
    case NBODY_OPT_STREAM:
      c->stream = value ? reinterpret_cast<cudaStream_t>(value) : c->own_stream;
      return NBODY_OK;
    case NBODY_OPT_USE_GRAPH:
      if (value != 0 && value != 1) return fail(c, NBODY_EINVAL, "use_graph must be 0 or 1");
      c->use_graph = value != 0;
      return NBODY_OK;
    case NBODY_OPT_BUILD:
      if (value < 0 || value > 1) return fail(c, NBODY_EINVAL, "unknown build variant");
      c->build_variant = int(value);
      drop_graph(c);
      return NBODY_OK;
    case NBODY_OPT_MULTIPOLE:
      if (value != 1 && value != 2) return fail(c, NBODY_EINVAL, "multipole order must be 1 or 2");
      if (value == 2 && c->f64) return fail(c, NBODY_EINVAL, "the FP64 mode is monopole only");
      if (value == 2 && c->traversal == 2) return fail(c, NBODY_EINVAL, "traversal variant 2 is monopole only");
      if (value == 2 && !c->tree.S64) {  // allocated on first use: 80 B per internal id
        const size_t inner = size_t(1) << c->tree.L;
        const nbody_status st = dev_alloc(c, quad_bytes_for(c->n), &c->quad_arena, "quadrupole arrays");
        if (st != NBODY_OK) return st;
        c->tree.S64 = reinterpret_cast<Quad64*>(c->quad_arena);
        c->tree.qf = reinterpret_cast<float4*>(static_cast<char*>(c->quad_arena) + 48 * inner);
      }
      c->tree.quad = value == 2;
      drop_graph(c);
      return NBODY_OK;
    case NBODY_OPT_SORT_EVERY:
      if (value < 1 || value > (int64_t(1) << 30)) return fail(c, NBODY_EINVAL, "sort_every must be >= 1");
      c->sort_every = int(value);
      return NBODY_OK;
    case NBODY_OPT_TIMING:
      if (value != 0 && value != 1) return fail(c, NBODY_EINVAL, "timing must be 0 or 1");
      c->timing = value != 0;
      return NBODY_OK;
    case NBODY_OPT_PRECISION: {
      if (value != 32 && value != 64) return fail(c, NBODY_EINVAL, "precision must be 32 or 64");
      const bool want = value == 64;
      if (want && (c->world > 1 || c->xpeer))
        return fail(c, NBODY_EINVAL, "the FP64 mode runs on a single rank (no exchange)");
      if (want && (c->tree.quad || c->traversal != 0))
        return fail(c, NBODY_EINVAL, "the FP64 mode needs monopole order and traversal variant 0");
      if (want && !c->arena64) {
        const nbody_status st = alloc_f64(c);
        if (st != NBODY_OK) return st;
      }
      c->f64 = want;
      c->tree.rec64 = want ? c->pm64[1] - (int64_t(1) << c->tree.L) : nullptr;
      c->loaded = false;  // bodies must be (re)loaded in the new precision
      c->have_force = false;
      drop_graph(c);
      return NBODY_OK;
    }
    case NBODY_OPT_BALANCE:
      if (value != 0 && value != 1) return fail(c, NBODY_EINVAL, "balance must be 0 or 1");
      c->balance = value != 0;
      drop_graph(c);
      return NBODY_OK;
    case NBODY_OPT_TRAVERSAL:
      if (value < 0 || value > 2) return fail(c, NBODY_EINVAL, "unknown traversal variant");
      if (value != 0 && c->f64) return fail(c, NBODY_EINVAL, "the FP64 mode uses traversal variant 0");
      if (value == 2 && c->tree.quad) return fail(c, NBODY_EINVAL, "traversal variant 2 is monopole only");
      c->traversal = int(value);
      drop_graph(c);
      return NBODY_OK;
    default:
      return fail(c, NBODY_EINVAL, "unknown option " + std::to_string(option));
  }
}

nbody_status nbody_set_bodies64(nbody_ctx* c, const double* pos, const double* vel, const double* mass) {
  CHECK_CTX(c);
  if (!c->f64) return fail(c, NBODY_EINVAL, "nbody_set_bodies64 needs NBODY_OPT_PRECISION = 64");
  if (!pos || !vel || !mass) return fail(c, NBODY_EINVAL, "null input");
  const int64_t n = c->n;
  const double *dp = pos, *dv = vel, *dm = mass;
  cudaStream_t s = c->stream;
  // host inputs go through buffers that the next pass overwrites anyway
  if (!is_device_ptr(pos)) {
    CK(cudaMemcpyAsync(c->acc64, pos, 24 * size_t(n), cudaMemcpyDefault, s));
    dp = reinterpret_cast<const double*>(c->acc64);
  }
  if (!is_device_ptr(vel)) {
    CK(cudaMemcpyAsync(c->pm64[1], vel, 24 * size_t(n), cudaMemcpyDefault, s));
    dv = reinterpret_cast<const double*>(c->pm64[1]);
  }
  if (!is_device_ptr(mass)) {
    CK(cudaMemcpyAsync(c->vi64[1], mass, 8 * size_t(n), cudaMemcpyDefault, s));
    dm = reinterpret_cast<const double*>(c->vi64[1]);
  }
  CK(cudaMemsetAsync(c->bad, 0, sizeof(int), s));
  launch_pack_bodies_f64(dp, dv, dm, n, c->pm64[0], c->vi64[0], c->bad, s);
  CK(cudaGetLastError());
  int bad = 0;
  CK(cudaMemcpyAsync(&bad, c->bad, sizeof(int), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (bad) {
    c->loaded = false;
    return fail(c, NBODY_EINVAL, (bad & 2) ? "masses must be finite and > 0" : "non-finite position or velocity");
  }
  c->loaded = true;
  c->have_force = false;
  c->keys_dbg_valid = false;
  c->steps = 0;
  return NBODY_OK;
}

nbody_status nbody_set_bodies(nbody_ctx* c, const float* pos, const float* vel, const float* mass) {
  CHECK_CTX(c);
  if (c->f64) return fail(c, NBODY_EINVAL, "FP64 mode: use nbody_set_bodies64");
  if (!pos || !vel || !mass) return fail(c, NBODY_EINVAL, "null input");
  const int64_t n = c->n;
  const float *dp = pos, *dv = vel, *dm = mass;
  cudaStream_t s = c->stream;
  // host inputs are staged in buffers only this rank reads (peers read acc
  // and cnt directly in the peer-exchange mode)
  if (!is_device_ptr(pos)) {
    CK(cudaMemcpyAsync(c->stage, pos, 12 * size_t(n), cudaMemcpyDefault, s));
    dp = reinterpret_cast<const float*>(c->stage);
  }
  if (!is_device_ptr(vel)) {
    CK(cudaMemcpyAsync(c->out3, vel, 12 * size_t(n), cudaMemcpyDefault, s));
    dv = c->out3;
  }
  if (!is_device_ptr(mass)) {
    CK(cudaMemcpyAsync(c->stage2, mass, 4 * size_t(n), cudaMemcpyDefault, s));
    dm = reinterpret_cast<const float*>(c->stage2);
  }
  CK(cudaMemsetAsync(c->bad, 0, sizeof(int), s));
  launch_pack_bodies(dp, dv, dm, n, c->pm[0], c->vi[0], c->bad, s);
  launch_bbox_partial(c->pm[0], n, c->bbox_part, c->nbbox, s);  // S1 partials of the new state
  CK(cudaGetLastError());
  int bad = 0;
  CK(cudaMemcpyAsync(&bad, c->bad, sizeof(int), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (bad) {
    c->loaded = false;
    return fail(c, NBODY_EINVAL, (bad & 2) ? "masses must be finite and > 0" : "non-finite position or velocity");
  }
  c->loaded = true;
  c->have_force = false;
  c->keys_dbg_valid = false;
  c->steps = 0;
  return NBODY_OK;
}

// Restore a slot-order state written by nbody_get_state(64) (checkpoint /
// resume): the records go straight into the current-state buffers, so the
// slot order -- which decides the stable sort's tie order (Alg. 7, [A10]) --
// and the ids survive, and the step counter restores the tree-reuse phase.
static nbody_status set_state_common(nbody_ctx* c, const void* pos_m, const void* vel_id, int64_t steps,
                                     size_t rec) {
  if (!pos_m || !vel_id) return fail(c, NBODY_EINVAL, "null input");
  if (steps < 0) return fail(c, NBODY_EINVAL, "steps < 0");
  const int64_t n = c->n;
  cudaStream_t s = c->stream;
  void* pm = c->f64 ? static_cast<void*>(c->pm64[0]) : static_cast<void*>(c->pm[0]);
  void* vi = c->f64 ? static_cast<void*>(c->vi64[0]) : static_cast<void*>(c->vi[0]);
  CK(cudaMemcpyAsync(pm, pos_m, rec * size_t(n), cudaMemcpyDefault, s));
  CK(cudaMemcpyAsync(vi, vel_id, rec * size_t(n), cudaMemcpyDefault, s));
  CK(cudaMemsetAsync(c->bad, 0, sizeof(int), s));
  CK(cudaMemsetAsync(c->idx[1], 0, sizeof(uint32_t) * size_t(n), s));  // id claims (the sort rewrites idx)
  if (c->f64) {
    launch_check_state_f64(c->pm64[0], c->vi64[0], n, c->idx[1], c->bad, s);
  } else {
    launch_check_state(c->pm[0], c->vi[0], n, c->idx[1], c->bad, s);
    launch_bbox_partial(c->pm[0], n, c->bbox_part, c->nbbox, s);  // S1 partials of the restored state
  }
  CK(cudaGetLastError());
  int bad = 0;
  CK(cudaMemcpyAsync(&bad, c->bad, sizeof(int), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  c->have_force = false;
  c->keys_dbg_valid = false;
  if (bad) {
    c->loaded = false;
    return fail(c, NBODY_EINVAL, (bad & 4) ? "state ids are not a permutation of [0, n)"
                                 : (bad & 2) ? "masses must be finite and > 0"
                                             : "non-finite position or velocity");
  }
  c->loaded = true;
  c->steps = steps;
  return NBODY_OK;
}

nbody_status nbody_set_state(nbody_ctx* c, const float* pos_m, const float* vel_id, int64_t steps) {
  CHECK_CTX(c);
  if (c->f64) return fail(c, NBODY_EINVAL, "FP64 mode: use nbody_set_state64");
  return set_state_common(c, pos_m, vel_id, steps, sizeof(float4));
}

nbody_status nbody_set_state64(nbody_ctx* c, const double* pos_m, const double* vel_id, int64_t steps) {
  CHECK_CTX(c);
  if (!c->f64) return fail(c, NBODY_EINVAL, "nbody_set_state64 needs NBODY_OPT_PRECISION = 64");
  return set_state_common(c, pos_m, vel_id, steps, sizeof(double4));
}

// Lazily create the copy stream, events and staging buffers of the
// pipelined transfers.
static nbody_status ensure_xfer(nbody_ctx* c) {
  if (c->xfer) return NBODY_OK;
  const size_t n = size_t(c->n);
  if (!c->cstream) CK(cudaStreamCreateWithFlags(&c->cstream, cudaStreamNonBlocking));
  if (!c->ostream) CK(cudaStreamCreateWithFlags(&c->ostream, cudaStreamNonBlocking));
  for (int k = 0; k < 2; ++k)
    for (cudaEvent_t* e : {&c->ev_in_copied[k], &c->ev_in_used[k], &c->ev_out_ready[k], &c->ev_out_copied[k]})
      if (!*e) CK(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
  void* p = nullptr;
  const nbody_status st = dev_alloc(c, xfer_bytes_for(c->n), &p, "staging buffers of the pipelined transfers");
  if (st != NBODY_OK) return st;
  c->xfer = static_cast<char*>(p);
  c->bad_async = reinterpret_cast<int*>(c->xfer + align_up(2 * 28 * n) + align_up(2 * 12 * n));
  CK(cudaMemsetAsync(c->bad_async, 0, sizeof(int), c->stream));
  return NBODY_OK;
}

nbody_status nbody_set_bodies_async(nbody_ctx* c, const float* pos, const float* vel, const float* mass) {
  CHECK_CTX(c);
  if (c->f64) return fail(c, NBODY_EINVAL, "FP64 mode: use nbody_set_bodies64");
  if (!pos || !vel || !mass) return fail(c, NBODY_EINVAL, "null input");
  nbody_status st = ensure_xfer(c);
  if (st != NBODY_OK) return st;
  const size_t n = size_t(c->n);
  const int k = c->slot_in;
  c->slot_in ^= 1;
  float* in = reinterpret_cast<float*>(c->xfer + k * 28 * n);
  // the staging buffer is free once the packing of the set before last ran
  if (c->ev_in_used_rec[k]) CK(cudaStreamWaitEvent(c->cstream, c->ev_in_used[k], 0));
  CK(cudaMemcpyAsync(in, pos, 12 * n, cudaMemcpyDefault, c->cstream));
  CK(cudaMemcpyAsync(in + 3 * n, vel, 12 * n, cudaMemcpyDefault, c->cstream));
  CK(cudaMemcpyAsync(in + 6 * n, mass, 4 * n, cudaMemcpyDefault, c->cstream));
  CK(cudaEventRecord(c->ev_in_copied[k], c->cstream));
  CK(cudaStreamWaitEvent(c->stream, c->ev_in_copied[k], 0));
  launch_pack_bodies(in, in + 3 * n, in + 6 * n, c->n, c->pm[0], c->vi[0], c->bad_async, c->stream);
  launch_bbox_partial(c->pm[0], c->n, c->bbox_part, c->nbbox, c->stream);  // S1 partials of the new state
  CK(cudaGetLastError());
  CK(cudaEventRecord(c->ev_in_used[k], c->stream));
  c->ev_in_used_rec[k] = true;
  c->loaded = true;
  c->have_force = false;
  c->keys_dbg_valid = false;
  c->steps = 0;
  return NBODY_OK;
}

nbody_status nbody_get_positions_async(nbody_ctx* c, float* out) {
  CHECK_CTX(c);
  if (c->f64) return fail(c, NBODY_EINVAL, "FP64 mode: use nbody_get_positions64");
  if (!out) return fail(c, NBODY_EINVAL, "null output");
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  nbody_status st = ensure_xfer(c);
  if (st != NBODY_OK) return st;
  const size_t n = size_t(c->n);
  const int k = c->slot_out;
  c->slot_out ^= 1;
  float* stage = reinterpret_cast<float*>(c->xfer + align_up(2 * 28 * n) + k * 12 * n);
  // the staging buffer is free once the copy-out issued two calls ago is done
  if (c->ev_out_copied_rec[k]) CK(cudaStreamWaitEvent(c->stream, c->ev_out_copied[k], 0));
  launch_scatter_by_id3(c->pm[0], c->vi[0], c->n, stage, c->stream);
  CK(cudaGetLastError());
  CK(cudaEventRecord(c->ev_out_ready[k], c->stream));
  CK(cudaStreamWaitEvent(c->ostream, c->ev_out_ready[k], 0));
  CK(cudaMemcpyAsync(out, stage, 12 * n, cudaMemcpyDefault, c->ostream));
  CK(cudaEventRecord(c->ev_out_copied[k], c->ostream));
  c->ev_out_copied_rec[k] = true;
  return NBODY_OK;
}

nbody_status nbody_compute_accel(nbody_ctx* c) {
  nvtxRangePushA("nbody_compute_accel");
  struct Pop { ~Pop() { nvtxRangePop(); } } pop_;
  CHECK_CTX(c);
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  nbody_status s = enqueue_pass(c, c->stream, false, true);
  if (s != NBODY_OK) return s;
  c->have_force = true;
  c->keys_dbg_valid = true;
  c->steps += 0;
  return NBODY_OK;
}

struct NvtxScope {
  explicit NvtxScope(const char* name) { nvtxRangePushA(name); }
  ~NvtxScope() { nvtxRangePop(); }
};

nbody_status nbody_step(nbody_ctx* c, int nsteps) {
  NvtxScope nv("nbody_step");
  CHECK_CTX(c);
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  if (nsteps < 0) return fail(c, NBODY_EINVAL, "nsteps < 0");
  if (nsteps == 0) return NBODY_OK;
  for (int i = 0; i < nsteps; ++i) {
    // step k of this body set re-sorts iff k % sort_every == 0 (always the first)
    const bool resort = (c->steps + i) % c->sort_every == 0;
    if (c->use_graph) {
      cudaGraphExec_t& exec = resort ? c->gexec : c->gexec_reuse;
      if (!exec) {
        nbody_status s = build_graph(c, resort);
        if (s != NBODY_OK) return s;
      }
      CK(cudaGraphLaunch(exec, c->stream));
      c->ev_valid = false;
    } else {
      nbody_status s = enqueue_pass(c, c->stream, true, false, resort);
      if (s != NBODY_OK) return s;
    }
    c->last_sorted = resort;
  }
  c->have_force = true;
  c->keys_dbg_valid = false;
  c->steps += nsteps;
  return NBODY_OK;
}

nbody_status nbody_sync(nbody_ctx* c) {
  CHECK_CTX(c);
  if (c->cstream) CK(cudaStreamSynchronize(c->cstream));
  if (c->ostream) CK(cudaStreamSynchronize(c->ostream));
  const nbody_status st = sync_stream(c);
  if (st != NBODY_OK || !c->bad_async) return st;
  int bad = 0;
  CK(cudaMemcpyAsync(&bad, c->bad_async, sizeof(int), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  if (bad) {
    CK(cudaMemsetAsync(c->bad_async, 0, sizeof(int), c->stream));
    c->loaded = false;
    return fail(c, NBODY_EINVAL, (bad & 2) ? "an async input set had masses that are not finite and > 0"
                                           : "an async input set had a non-finite position or velocity");
  }
  return NBODY_OK;
}

// out[id][3] <- src[i].xyz for the slots [b, e) (src[i] belongs to slot b + i).
// A host `out` goes through the device staging buffer out3.
// Peer-exchange mode: copy every rank's owned slice of a per-rank array
// (acc or cnt, indexed from the owner's first slot) into dst by slot.
static nbody_status gather_peers(nbody_ctx* c, const void* const* src, void* dst, size_t rec_bytes) {
  for (int q = 0; q < c->world; ++q) {
    int64_t b = 0, e = 0;
    const nbody_status st = rank_range(c, q, &b, &e);
    if (st != NBODY_OK) return st;
    if (e > b)
      CK(cudaMemcpyAsync(static_cast<char*>(dst) + rec_bytes * size_t(b), src[q], rec_bytes * size_t(e - b),
                         cudaMemcpyDefault, c->stream));
  }
  return NBODY_OK;
}

static nbody_status get_by_id3(nbody_ctx* c, const float4* src, int64_t b, int64_t e, float* out) {
  if (!out) return fail(c, NBODY_EINVAL, "null output");
  const int64_t n = c->n;
  const bool dev = is_device_ptr(out);
  float* dst = dev ? out : c->out3;
  if (!dev && (b > 0 || e < n)) CK(cudaMemcpyAsync(dst, out, 12 * size_t(n), cudaMemcpyDefault, c->stream));
  launch_scatter_by_id3(src, c->vi[0] + b, e - b, dst, c->stream);
  CK(cudaGetLastError());
  if (!dev) CK(cudaMemcpyAsync(out, dst, 12 * size_t(n), cudaMemcpyDefault, c->stream));
  return sync_stream(c);
}

// NEXT-2 FP64 mode: out[id][3] <- src[slot].xyz for all slots (fp64, or
// rounded to fp32 for the fp32 getters).
static nbody_status get_by_id3_f64(nbody_ctx* c, const double4* src, void* out, bool as_f32) {
  if (!out) return fail(c, NBODY_EINVAL, "null output");
  const int64_t n = c->n;
  const bool dev = is_device_ptr(out);
  void* dst = dev ? out : static_cast<void*>(c->stage64);
  if (as_f32)
    launch_scatter_by_id3_f64to32(src, c->vi64[0], n, static_cast<float*>(dst), c->stream);
  else
    launch_scatter_by_id3_f64(src, c->vi64[0], n, static_cast<double*>(dst), c->stream);
  CK(cudaGetLastError());
  if (!dev) CK(cudaMemcpyAsync(out, dst, (as_f32 ? 12 : 24) * size_t(n), cudaMemcpyDefault, c->stream));
  return sync_stream(c);
}

#ifdef NBODY_WITH_NCCL
// Collective: gather every rank's owned slice of src (S records of `words`
// 4-byte words) into dst, indexed by slot.
static nbody_status gather_owned(nbody_ctx* c, const void* src, void* dst, size_t words) {
  const ncclResult_t r = ncclAllGather(src, dst, words * size_t(c->own_s), ncclFloat, c->comm, c->stream);
  if (r != ncclSuccess) return fail(c, NBODY_ENCCL, ncclGetErrorString(r));
  return NBODY_OK;
}
#endif

nbody_status nbody_get_accel(nbody_ctx* c, float* out) {
  CHECK_CTX(c);
  if (!c->have_force) return fail(c, NBODY_ESTATE, "no force pass yet");
  if (c->f64) return get_by_id3_f64(c, c->acc64, out, true);
#ifdef NBODY_WITH_NCCL
  if (c->comm) {
    nbody_status s = gather_owned(c, c->acc, c->stage, 4);
    if (s != NBODY_OK) return s;
    return get_by_id3(c, c->stage, 0, c->n, out);
  }
#endif
  if (c->xpeer) {
    nbody_status s = gather_peers(c, reinterpret_cast<const void* const*>(c->peer_acc), c->stage, 16);
    if (s != NBODY_OK) return s;
    return get_by_id3(c, c->stage, 0, c->n, out);
  }
  return get_by_id3(c, c->acc, c->own_b, c->own_e, out);
}

nbody_status nbody_get_positions(nbody_ctx* c, float* out) {
  CHECK_CTX(c);
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  if (c->f64) return get_by_id3_f64(c, c->pm64[0], out, true);
  return get_by_id3(c, c->pm[0], 0, c->n, out);
}

nbody_status nbody_get_velocities(nbody_ctx* c, float* out) {
  CHECK_CTX(c);
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  if (c->f64) return get_by_id3_f64(c, c->vi64[0], out, true);
  return get_by_id3(c, c->vi[0], 0, c->n, out);
}

nbody_status nbody_get_positions64(nbody_ctx* c, double* out) {
  CHECK_CTX(c);
  if (!c->f64) return fail(c, NBODY_EINVAL, "needs NBODY_OPT_PRECISION = 64");
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  return get_by_id3_f64(c, c->pm64[0], out, false);
}

nbody_status nbody_get_velocities64(nbody_ctx* c, double* out) {
  CHECK_CTX(c);
  if (!c->f64) return fail(c, NBODY_EINVAL, "needs NBODY_OPT_PRECISION = 64");
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  return get_by_id3_f64(c, c->vi64[0], out, false);
}

nbody_status nbody_get_accel64(nbody_ctx* c, double* out) {
  CHECK_CTX(c);
  if (!c->f64) return fail(c, NBODY_EINVAL, "needs NBODY_OPT_PRECISION = 64");
  if (!c->have_force) return fail(c, NBODY_ESTATE, "no force pass yet");
  return get_by_id3_f64(c, c->acc64, out, false);
}

nbody_status nbody_get_interactions(nbody_ctx* c, uint32_t* out) {
  CHECK_CTX(c);
  if (!c->have_force) return fail(c, NBODY_ESTATE, "no force pass yet");
  if (!out) return fail(c, NBODY_EINVAL, "null output");
  const int64_t n = c->n;
  const uint32_t* src = c->cnt;
  int64_t b = c->own_b, e = c->own_e;
#ifdef NBODY_WITH_NCCL
  if (c->comm) {
    nbody_status s = gather_owned(c, c->cnt, c->stage2, 1);
    if (s != NBODY_OK) return s;
    src = c->stage2;
    b = 0;
    e = n;
  }
#endif
  if (c->xpeer) {
    nbody_status s = gather_peers(c, reinterpret_cast<const void* const*>(c->peer_cnt), c->stage2, 4);
    if (s != NBODY_OK) return s;
    src = c->stage2;
    b = 0;
    e = n;
  }
  const bool dev = is_device_ptr(out);
  uint32_t* dst = dev ? out : reinterpret_cast<uint32_t*>(c->out3);
  if (!dev && (b > 0 || e < n)) CK(cudaMemcpyAsync(dst, out, 4 * size_t(n), cudaMemcpyDefault, c->stream));
  if (c->f64)
    launch_scatter_by_id1_f64(src, c->vi64[0] + b, e - b, dst, c->stream);
  else
    launch_scatter_by_id1(src, c->vi[0] + b, e - b, dst, c->stream);
  CK(cudaGetLastError());
  if (!dev) CK(cudaMemcpyAsync(out, dst, 4 * size_t(n), cudaMemcpyDefault, c->stream));
  return sync_stream(c);
}

// ---- NEXT-1: all-pairs reference ------------------------------------------

nbody_status nbody_direct_accel(nbody_ctx* c, const int64_t* ids, int64_t nt, double* out) {
  CHECK_CTX(c);
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  if (nt < 0 || (nt > 0 && (!ids || !out))) return fail(c, NBODY_EINVAL, "bad target list");
  if (c->f64) return fail(c, NBODY_EINVAL, "nbody_direct_accel works on the fp32 state (precision 32)");
  if (nt == 0) return NBODY_OK;
  const bool ids_dev = is_device_ptr(ids);
  if (!ids_dev)
    for (int64_t i = 0; i < nt; ++i)
      if (ids[i] < 0 || ids[i] >= c->n) return fail(c, NBODY_EINVAL, "id out of range");
  const int64_t chunks = direct_chunks(c->n, nt);
  cudaStream_t s = c->stream;
  char* tmp = nullptr;
  const size_t bi = align_up(8 * size_t(nt)), bt = align_up(4 * size_t(nt)), bp = align_up(32 * size_t(chunks * nt));
  const size_t bo = align_up(24 * size_t(nt));
  CK(cudaMallocAsync(reinterpret_cast<void**>(&tmp), bi + bt + bp + bo, s));
  int64_t* d_ids = reinterpret_cast<int64_t*>(tmp);
  uint32_t* d_tslot = reinterpret_cast<uint32_t*>(tmp + bi);
  double4* d_part = reinterpret_cast<double4*>(tmp + bi + bt);
  double* d_out = reinterpret_cast<double*>(tmp + bi + bt + bp);
  cudaError_t e = cudaMemcpyAsync(d_ids, ids, 8 * size_t(nt), cudaMemcpyDefault, s);
  if (e == cudaSuccess) {
    launch_direct(c->pm[0], c->vi[0], c->n, d_ids, nt, c->eps * c->eps, c->stage2, d_tslot, d_part, d_out, s);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaMemcpyAsync(out, d_out, 24 * size_t(nt), cudaMemcpyDefault, s);
  cudaFreeAsync(tmp, s);
  if (e != cudaSuccess) return fail(c, NBODY_ECUDA, cudaGetErrorString(e));
  return sync_stream(c);
}

nbody_status nbody_allpairs_accel(nbody_ctx* c, const int64_t* ids, int64_t nt, double* out, float* kernel_ms) {
  CHECK_CTX(c);
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  if (nt < 0 || (nt > 0 && (!ids || !out))) return fail(c, NBODY_EINVAL, "bad target list");
  if (c->f64) return fail(c, NBODY_EINVAL, "nbody_allpairs_accel works on the fp32 state (precision 32)");
  if (kernel_ms) *kernel_ms = 0.f;
  if (nt == 0) return NBODY_OK;
  const bool ids_dev = is_device_ptr(ids);
  if (!ids_dev)
    for (int64_t i = 0; i < nt; ++i)
      if (ids[i] < 0 || ids[i] >= c->n) return fail(c, NBODY_EINVAL, "id out of range");
  const int64_t chunks = allpairs_chunks(c->n, nt, c->nsm);
  cudaStream_t s = c->stream;
  char* tmp = nullptr;
  const size_t bi = align_up(8 * size_t(nt)), bt = align_up(4 * size_t(nt)), bp = align_up(32 * size_t(chunks * nt));
  const size_t bo = align_up(24 * size_t(nt));
  CK(cudaMallocAsync(reinterpret_cast<void**>(&tmp), bi + bt + bp + bo, s));
  int64_t* d_ids = reinterpret_cast<int64_t*>(tmp);
  uint32_t* d_tslot = reinterpret_cast<uint32_t*>(tmp + bi);
  double4* d_part = reinterpret_cast<double4*>(tmp + bi + bt);
  double* d_out = reinterpret_cast<double*>(tmp + bi + bt + bp);
  cudaError_t e = cudaMemcpyAsync(d_ids, ids, 8 * size_t(nt), cudaMemcpyDefault, s);
  if (e == cudaSuccess) {
    launch_target_slots(c->vi[0], c->n, d_ids, nt, c->stage2, d_tslot, s);
    launch_allpairs32(c->pm[0], c->n, d_tslot, nt, float(c->eps * c->eps), chunks, d_part, d_out,
                      kernel_ms ? c->ev[0] : nullptr, kernel_ms ? c->ev[1] : nullptr, s);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaMemcpyAsync(out, d_out, 24 * size_t(nt), cudaMemcpyDefault, s);
  cudaFreeAsync(tmp, s);
  if (e != cudaSuccess) return fail(c, NBODY_ECUDA, cudaGetErrorString(e));
  const nbody_status st = sync_stream(c);
  if (st != NBODY_OK) return st;
  if (kernel_ms) CK(cudaEventElapsedTime(kernel_ms, c->ev[0], c->ev[1]));
  c->ev_valid = false;  // the stage events now hold the all-pairs kernel
  return NBODY_OK;
}

// ---- partition / multi-GPU -------------------------------------------------

nbody_status nbody_set_partition(nbody_ctx* c, int rank, int world) {
  CHECK_CTX(c);
  if (world < 1 || world > kMaxWorld || rank < 0 || rank >= world)
    return fail(c, NBODY_EINVAL, "need 0 <= rank < world <= 256");
  if (c->f64 && world > 1) return fail(c, NBODY_EINVAL, "the FP64 mode runs on a single rank");
#ifdef NBODY_WITH_NCCL
  if (c->comm) return fail(c, NBODY_ESTATE, "a communicator is attached");
#endif
  if (c->xpeer) return fail(c, NBODY_ESTATE, "peers are attached");
  set_part(c, rank, world);
  drop_graph(c);
  return NBODY_OK;
}

nbody_status nbody_get_partition(nbody_ctx* c, int* rank, int* world, int64_t* begin, int64_t* end) {
  CHECK_CTX(c);
  if (rank) *rank = c->rank;
  if (world) *world = c->world;
  int64_t b = c->own_b, e = c->own_e;
  if (balanced(c)) {  // NEXT-3(i): the range of the last force pass
    const nbody_status st = rank_range(c, c->rank, &b, &e);
    if (st != NBODY_OK) return st;
  }
  if (begin) *begin = b;
  if (end) *end = e;
  return NBODY_OK;
}

nbody_status nbody_copy_owned(nbody_ctx* dst, nbody_ctx* src) {
  CHECK_CTX(dst);
  nbody_ctx* c = dst;
  if (!src || src->n != dst->n || src->world != dst->world) return fail(c, NBODY_EINVAL, "incompatible contexts");
  const int64_t b = src->own_b, len = src->own_e - src->own_b;
  if (len <= 0) return NBODY_OK;
  CK(cudaStreamSynchronize(src->stream));
  CK(cudaMemcpyAsync(dst->pm[0] + b, src->pm[0] + b, 16 * size_t(len), cudaMemcpyDeviceToDevice, dst->stream));
  CK(cudaMemcpyAsync(dst->vi[0] + b, src->vi[0] + b, 16 * size_t(len), cudaMemcpyDeviceToDevice, dst->stream));
  return sync_stream(dst);
}

nbody_status nbody_partition(int64_t n, int rank, int world, int64_t* begin, int64_t* end) {
  if (n < 1 || world < 1 || world > kMaxWorld || rank < 0 || rank >= world || !begin || !end) return NBODY_EINVAL;
  nbody_ctx tmp;
  tmp.n = n;
  set_part(&tmp, rank, world);
  *begin = tmp.own_b;
  *end = tmp.own_e;
  return NBODY_OK;
}

int nbody_has_nccl(void) {
#ifdef NBODY_WITH_NCCL
  return 1;
#else
  return 0;
#endif
}

nbody_status nbody_nccl_unique_id(void* out) {
  if (!out) return NBODY_EINVAL;
#ifdef NBODY_WITH_NCCL
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return NBODY_ENCCL;
  std::memcpy(out, &id, sizeof(id));
  return NBODY_OK;
#else
  return NBODY_ENCCL;
#endif
}

nbody_status nbody_attach_nccl(nbody_ctx* c, const void* unique_id, int rank, int world) {
  CHECK_CTX(c);
  if (!unique_id || world < 1 || world > kMaxWorld || rank < 0 || rank >= world)
    return fail(c, NBODY_EINVAL, "need a unique id and 0 <= rank < world <= 256");
  if (c->f64) return fail(c, NBODY_EINVAL, "the FP64 mode runs on a single rank");
#ifdef NBODY_WITH_NCCL
  if (c->comm) return fail(c, NBODY_ESTATE, "a communicator is already attached");
  if (c->xpeer) return fail(c, NBODY_ESTATE, "peers are attached");
  ncclUniqueId id;
  std::memcpy(&id, unique_id, sizeof(id));
  const ncclResult_t r = ncclCommInitRank(&c->comm, world, id, rank);
  if (r != ncclSuccess) {
    c->comm = nullptr;
    return fail(c, NBODY_ENCCL, std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
  }
  set_part(c, rank, world);
  drop_graph(c);
  return NBODY_OK;
#else
  return fail(c, NBODY_ENCCL, "library built without NCCL");
#endif
}

nbody_status nbody_attach_comm(nbody_ctx* c, void* nccl_comm, int rank, int world) {
  CHECK_CTX(c);
  if (!nccl_comm || world < 1 || world > kMaxWorld || rank < 0 || rank >= world)
    return fail(c, NBODY_EINVAL, "need a communicator and 0 <= rank < world <= 256");
  if (c->f64) return fail(c, NBODY_EINVAL, "the FP64 mode runs on a single rank");
#ifdef NBODY_WITH_NCCL
  if (c->comm) return fail(c, NBODY_ESTATE, "a communicator is already attached");
  if (c->xpeer) return fail(c, NBODY_ESTATE, "peers are attached");
  ncclComm_t comm = static_cast<ncclComm_t>(nccl_comm);
  int r = -1, w = -1, d = -1;
  ncclResult_t e = ncclCommUserRank(comm, &r);
  if (e == ncclSuccess) e = ncclCommCount(comm, &w);
  if (e == ncclSuccess) e = ncclCommCuDevice(comm, &d);
  if (e != ncclSuccess) return fail(c, NBODY_ENCCL, std::string("communicator query: ") + ncclGetErrorString(e));
  if (r != rank || w != world)
    return fail(c, NBODY_EINVAL, "the communicator is rank " + std::to_string(r) + " of " + std::to_string(w));
  if (d != c->device) return fail(c, NBODY_EINVAL, "the communicator belongs to another device");
  c->comm = comm;
  c->comm_borrowed = true;
  set_part(c, rank, world);
  drop_graph(c);
  return NBODY_OK;
#else
  return fail(c, NBODY_ENCCL, "library built without NCCL");
#endif
}

// ---- fused exchange over peer memory --------------------------------------

nbody_status nbody_peer_handle(nbody_ctx* c, void* out) {
  CHECK_CTX(c);
  if (!out) return fail(c, NBODY_EINVAL, "null output");
  PeerDesc d{};
  const char* base = nullptr;
  const nbody_status st = alloc_base(c, c->arena, &base);
  if (st != NBODY_OK) return st;
  CK(cudaIpcGetMemHandle(&d.ipc, const_cast<char*>(base)));
  d.offset = uint64_t(c->arena - base);
  d.n = c->n;
  d.arena_bytes = c->arena_bytes;
  d.magic = kPeerMagic;
  CK(cudaDeviceGetPCIBusId(d.pci, sizeof(d.pci), c->device));
  std::memset(out, 0, 128);
  std::memcpy(out, &d, sizeof(d));
  return NBODY_OK;
}

static nbody_status check_attach(nbody_ctx* c, int rank, int world) {
  if (c && c->f64) return fail(c, NBODY_EINVAL, "the FP64 mode runs on a single rank");
  if (world < 1 || world > kMaxPeers || rank < 0 || rank >= world)
    return fail(c, NBODY_EINVAL, "peer exchange needs 0 <= rank < world <= 8");
  if (c->xpeer) return fail(c, NBODY_ESTATE, "peers are already attached");
#ifdef NBODY_WITH_NCCL
  if (c->comm) return fail(c, NBODY_ESTATE, "a communicator is attached");
#endif
  return NBODY_OK;
}

nbody_status nbody_attach_peers(nbody_ctx* c, const void* handles, int rank, int world) {
  CHECK_CTX(c);
  nbody_status st = check_attach(c, rank, world);
  if (st != NBODY_OK) return st;
  if (!handles) return fail(c, NBODY_EINVAL, "null handles");
  char* base[kMaxPeers] = {};
  for (int q = 0; q < world; ++q) {
    PeerDesc d;
    std::memcpy(&d, static_cast<const char*>(handles) + 128 * size_t(q), sizeof(d));
    if (d.magic != kPeerMagic || d.n != c->n || d.arena_bytes != c->arena_bytes)
      return fail(c, NBODY_EINVAL, "peer " + std::to_string(q) + ": descriptor does not match this context");
    if (q == rank) {
      base[q] = c->arena;
      continue;
    }
    auto unmap = [&]() {
      for (int k = 0; k < q; ++k)
        if (c->peer_map[k]) cudaIpcCloseMemHandle(c->peer_map[k]), c->peer_map[k] = nullptr;
    };
    // the peer's arena must be reachable by loads/stores from this device
    // (NVLink/NVSwitch or PCIe P2P); say so instead of faulting in K7
    d.pci[sizeof(d.pci) - 1] = 0;
    int pdev = -1;
    if (cudaDeviceGetByPCIBusId(&pdev, d.pci) != cudaSuccess) {
      cudaGetLastError();
      unmap();
      return fail(c, NBODY_EINVAL, "peer " + std::to_string(q) + ": device " + d.pci +
                                       " is not visible to this process (CUDA_VISIBLE_DEVICES must expose every "
                                       "rank's GPU for the peer exchange; use the NCCL exchange otherwise)");
    }
    if (pdev != c->device) {
      int ok = 0;
      CK(cudaDeviceCanAccessPeer(&ok, c->device, pdev));
      if (!ok) {
        unmap();
        return fail(c, NBODY_EINVAL, "peer " + std::to_string(q) + ": no peer access from device " +
                                         std::to_string(c->device) + " to device " + std::to_string(pdev) +
                                         " (use the NCCL exchange)");
      }
    }
    void* p = nullptr;
    const cudaError_t e = cudaIpcOpenMemHandle(&p, d.ipc, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      cudaGetLastError();
      unmap();
      return fail(c, NBODY_ECUDA, "cudaIpcOpenMemHandle(peer " + std::to_string(q) + "): " + cudaGetErrorString(e));
    }
    c->peer_map[q] = p;
    base[q] = static_cast<char*>(p) + d.offset;
  }
  return attach_peer_bases(c, base, rank, world);
}

nbody_status nbody_attach_peers_local(nbody_ctx** ctxs, int world) {
  if (!ctxs || world < 1 || world > kMaxPeers) return NBODY_EINVAL;
  for (int r = 0; r < world; ++r) {
    nbody_ctx* c = ctxs[r];
    CHECK_CTX(c);
    nbody_status st = check_attach(c, r, world);
    if (st != NBODY_OK) return st;
    if (c->n != ctxs[0]->n || c->arena_bytes != ctxs[0]->arena_bytes)
      return fail(c, NBODY_EINVAL, "contexts differ in N");
  }
  for (int r = 0; r < world; ++r)  // contexts on different devices: enable peer access
    for (int q = 0; q < world; ++q) {
      if (ctxs[r]->device == ctxs[q]->device) continue;
      nbody_ctx* c = ctxs[r];
      int prev = -1;
      CK(cudaGetDevice(&prev));
      CK(cudaSetDevice(c->device));
      const cudaError_t e = cudaDeviceEnablePeerAccess(ctxs[q]->device, 0);
      cudaSetDevice(prev);
      if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
      else if (e != cudaSuccess) return fail(c, NBODY_ECUDA, std::string("peer access: ") + cudaGetErrorString(e));
    }
  char* base[kMaxPeers] = {};
  for (int q = 0; q < world; ++q) base[q] = ctxs[q]->arena;
  for (int r = 0; r < world; ++r) {
    const nbody_status st = attach_peer_bases(ctxs[r], base, r, world);
    if (st != NBODY_OK) return st;
  }
  return NBODY_OK;
}

int nbody_exchange_mode(nbody_ctx* c) {
  if (!c) return -1;
  if (c->xpeer) return 2;
#ifdef NBODY_WITH_NCCL
  if (c->comm) return 1;
#endif
  return 0;
}

nbody_status nbody_get_state64(nbody_ctx* c, double* pos_m, double* vel_id) {
  CHECK_CTX(c);
  if (!c->f64) return fail(c, NBODY_EINVAL, "needs NBODY_OPT_PRECISION = 64");
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  if (pos_m) CK(cudaMemcpyAsync(pos_m, c->pm64[0], 32 * size_t(c->n), cudaMemcpyDefault, c->stream));
  if (vel_id) CK(cudaMemcpyAsync(vel_id, c->vi64[0], 32 * size_t(c->n), cudaMemcpyDefault, c->stream));
  return sync_stream(c);
}

nbody_status nbody_get_state(nbody_ctx* c, float* pos_m, float* vel_id) {
  CHECK_CTX(c);
  if (c->f64) return fail(c, NBODY_EINVAL, "FP64 mode: use nbody_get_state64");
  if (!c->loaded) return fail(c, NBODY_ESTATE, "no bodies loaded");
  if (pos_m) CK(cudaMemcpyAsync(pos_m, c->pm[0], 16 * size_t(c->n), cudaMemcpyDefault, c->stream));
  if (vel_id) CK(cudaMemcpyAsync(vel_id, c->vi[0], 16 * size_t(c->n), cudaMemcpyDefault, c->stream));
  return sync_stream(c);
}

nbody_status nbody_get_stats(nbody_ctx* c, nbody_stats* out) {
  CHECK_CTX(c);
  if (!out) return fail(c, NBODY_EINVAL, "null output");
  std::memset(out, 0, sizeof(*out));
  out->n = c->n;
  out->key_bits = c->b;
  out->levels = c->tree.L;
  out->steps = c->steps;
  if (c->have_force) {
    unsigned long long t = 0;
    CK(cudaMemcpyAsync(&t, c->total, sizeof(t), cudaMemcpyDeviceToHost, c->stream));
    nbody_status s = sync_stream(c);
    if (s != NBODY_OK) return s;
    out->interactions = t;
  }
  out->kernels_per_step = c->kernels_per_step;
  // lane utilisation of K6's dense phase, from the design counters
  // (NBODY_K6_STATS builds only; counters since the last reset): interacting
  // lanes / (32 x dense-list slots)
  out->lane_util = -1.f;
  {
    unsigned long long st[9];
    if (force_stats(st, 9, false) == 9) {
      const double slots = 32.0 * double(st[5] + st[6]);
      if (slots > 0) out->lane_util = float(double(st[7] + st[8]) / slots);
    }
  }
  if (c->ev_valid) {
    CK(cudaEventSynchronize(c->ev[5]));
    float* dst[5] = {&out->ms_bbox_keys, &out->ms_sort, &out->ms_build, &out->ms_force, &out->ms_update};
    for (int i = 0; i < 5; ++i) CK(cudaEventElapsedTime(dst[i], c->ev[i], c->ev[i + 1]));
  }
  return NBODY_OK;
}

nbody_status nbody_debug_keys(nbody_ctx* c, uint64_t* keys) {
  CHECK_CTX(c);
  if (!keys) return fail(c, NBODY_EINVAL, "null output");
  if (!c->keys_dbg_valid) return fail(c, NBODY_ESTATE, "keys are kept by nbody_compute_accel only");
  const int64_t n = c->n;
  if (c->key_bytes == 8) {
    CK(cudaMemcpyAsync(keys, c->keys_dbg, 8 * size_t(n), cudaMemcpyDefault, c->stream));
    return sync_stream(c);
  }
  // widen u32 keys on the host side of the copy
  uint32_t* tmp = new (std::nothrow) uint32_t[size_t(n)];
  if (!tmp) return fail(c, NBODY_ENOMEM, "host buffer");
  cudaError_t e = cudaMemcpyAsync(tmp, c->keys_dbg, 4 * size_t(n), cudaMemcpyDefault, c->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
  if (e != cudaSuccess) {
    delete[] tmp;
    return fail(c, NBODY_ECUDA, cudaGetErrorString(e));
  }
  const bool dev = is_device_ptr(keys);
  if (!dev) {
    for (int64_t i = 0; i < n; ++i) keys[i] = tmp[i];
    delete[] tmp;
    return NBODY_OK;
  }
  uint64_t* wide = new (std::nothrow) uint64_t[size_t(n)];
  if (!wide) {
    delete[] tmp;
    return fail(c, NBODY_ENOMEM, "host buffer");
  }
  for (int64_t i = 0; i < n; ++i) wide[i] = tmp[i];
  e = cudaMemcpyAsync(keys, wide, 8 * size_t(n), cudaMemcpyDefault, c->stream);  // stream-ordered, like every copy
  if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
  delete[] tmp;
  delete[] wide;
  if (e != cudaSuccess) return fail(c, NBODY_ECUDA, cudaGetErrorString(e));
  return NBODY_OK;
}

nbody_status nbody_debug_perm(nbody_ctx* c, uint32_t* perm) {
  CHECK_CTX(c);
  if (!perm) return fail(c, NBODY_EINVAL, "null output");
  if (!c->have_force) return fail(c, NBODY_ESTATE, "no force pass yet");
  if (!c->last_sorted) return fail(c, NBODY_ESTATE, "the last pass reused the tree order (no sort)");
  CK(cudaMemcpyAsync(perm, c->idx[c->perm_buf], 4 * size_t(c->n), cudaMemcpyDefault, c->stream));
  return sync_stream(c);
}

int nbody_debug_force_stats(uint64_t* out, int n) {
  if (!out || n <= 0) return 0;
  return force_stats(reinterpret_cast<unsigned long long*>(out), n);
}

nbody_status nbody_debug_quad(nbody_ctx* c, int level, double* S) {
  CHECK_CTX(c);
  if (level < 1 || level > c->tree.L) return fail(c, NBODY_EINVAL, "level out of range [1, L]");
  if (!S) return fail(c, NBODY_EINVAL, "null output");
  if (!c->tree.quad || !c->have_force) return fail(c, NBODY_ESTATE, "quadrupoles not enabled or not built");
  CK(cudaMemcpyAsync(S, c->tree.S64 + c->tree.off[level], 48 * size_t(c->tree.count[level]), cudaMemcpyDefault,
                     c->stream));
  return sync_stream(c);
}

nbody_status nbody_debug_level(nbody_ctx* c, int level, int64_t* count, double* pred, float* rec, float* box) {
  CHECK_CTX(c);
  if (level < 1 || level > c->tree.L) return fail(c, NBODY_EINVAL, "level out of range [1, L]");
  const int64_t cnt = c->tree.count[level];
  if (count) *count = cnt;
  if (!pred && !rec && !box) return NBODY_OK;
  if (!c->have_force) return fail(c, NBODY_ESTATE, "no force pass yet");
  const int64_t off = c->tree.off[level];
  cudaStream_t s = c->stream;
  if (pred) CK(cudaMemcpyAsync(pred, c->tree.pred + off, 32 * size_t(cnt), cudaMemcpyDefault, s));
  if (rec) CK(cudaMemcpyAsync(rec, c->tree.rec + off, 16 * size_t(cnt), cudaMemcpyDefault, s));
  if (box && c->f64) return fail(c, NBODY_EINVAL, "FP64 mode: fp64 boxes via nbody_debug_level64");
  if (box) {
    CK(cudaMemcpy2DAsync(box, 24, c->tree.blo + off, 16, 12, size_t(cnt), cudaMemcpyDefault, s));
    CK(cudaMemcpy2DAsync(box + 3, 24, c->tree.bhi + off, 16, 12, size_t(cnt), cudaMemcpyDefault, s));
  }
  return sync_stream(c);
}

nbody_status nbody_debug_level64(nbody_ctx* c, int level, int64_t* count, double* rec64, double* box64) {
  CHECK_CTX(c);
  if (!c->f64) return fail(c, NBODY_EINVAL, "needs NBODY_OPT_PRECISION = 64");
  if (level < 1 || level > c->tree.L) return fail(c, NBODY_EINVAL, "level out of range [1, L]");
  const int64_t cnt = c->tree.count[level];
  if (count) *count = cnt;
  if (!rec64 && !box64) return NBODY_OK;
  if (!c->have_force) return fail(c, NBODY_ESTATE, "no force pass yet");
  const int64_t off = c->tree.off[level];
  cudaStream_t s = c->stream;
  if (rec64) CK(cudaMemcpyAsync(rec64, c->tree.rec64 + off, 32 * size_t(cnt), cudaMemcpyDefault, s));
  if (box64) {
    CK(cudaMemcpy2DAsync(box64, 48, c->tree.blo64 + off, 32, 24, size_t(cnt), cudaMemcpyDefault, s));
    CK(cudaMemcpy2DAsync(box64 + 3, 48, c->tree.bhi64 + off, 32, 24, size_t(cnt), cudaMemcpyDefault, s));
  }
  return sync_stream(c);
}

const char* nbody_last_error(const nbody_ctx* c) {
  if (!c) return "null context";
  return c->err.c_str();
}

void nbody_destroy(nbody_ctx* c) {
  if (!c) return;
  if (c->stream) cudaStreamSynchronize(c->stream);
  drop_graph(c);
#ifdef NBODY_WITH_NCCL
  if (c->comm && !c->comm_borrowed) ncclCommDestroy(c->comm);
#endif
  for (auto& p : c->peer_map)
    if (p) cudaIpcCloseMemHandle(p);
  dev_free(c, c->arena);
  dev_free(c, c->quad_arena);
  dev_free(c, c->arena64);
  for (auto& e : c->ev)
    if (e) cudaEventDestroy(e);
  for (cudaStream_t cs : {c->cstream, c->ostream})
    if (cs) {
      cudaStreamSynchronize(cs);
      cudaStreamDestroy(cs);
    }
  for (int k = 0; k < 2; ++k)
    for (cudaEvent_t e : {c->ev_in_copied[k], c->ev_in_used[k], c->ev_out_ready[k], c->ev_out_copied[k]})
      if (e) cudaEventDestroy(e);
  dev_free(c, c->xfer);
  if (c->cap_stream) cudaStreamDestroy(c->cap_stream);
  if (c->own_stream) cudaStreamDestroy(c->own_stream);
  cudaGetLastError();
  delete c;
}

}  // extern "C"
