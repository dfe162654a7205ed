// internal.cuh -- device data layout and kernel launchers of the B200 path.
//
// Product code only: nothing here is shared with oracle/ (DESIGN.md
// "Independence").  P:NNN = line of the paper text; [A#] = DESIGN.md reading.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace nb {

constexpr int kMaxLevels = 32;   // L = ceil(log2 N) <= 30 for N < 2^30
constexpr int kNumSMs = 148;     // B200; the engine re-reads the device's count

// Grid of the Hilbert quantisation computed on the device each step
// from the bounding box (Alg. 3).
struct GridInfo {
  float lo[3];
  float hi[3];
  double inv;    // 2^b / ext, or 0 when ext == 0 [A17]
  int b;         // bits per axis
  float abs_d2;  // absolute slack of the fp32 opening-test filter: 1e-9 R^2,
                 // R = max |coordinate| (K6)
  float R;       // max |coordinate| of this step's bodies (T-filter slack)
  double lo64[3];  // NEXT-2 FP64 mode: the fp64 bounding box (lo/hi unused)
  double hi64[3];
};

// NEXT-4 [A24]: second mass moment about the COM, S = sum m (x-c)(x-c)^T.
struct Quad64 {
  double s[6];  // xx, yy, zz, xy, xz, yz (fp64, build + debug)
};

// Balanced, ragged BVH in heap numbering ([A6]): node (l, j) has id
// off[l] + j with off[l] = 2^(L-l); leaf i is 2^L + i.
struct TreeView {
  int L;                       // levels above the leaves
  int64_t n;                   // bodies (= nodes at level 0)
  int64_t count[kMaxLevels];   // nodes per level: ceil(n / 2^l)
  int64_t off[kMaxLevels];     // start of level l in the node arrays
  double4* pred;   // (com64 x, y, z, s^2)   opening test data, fp64 [A3][A16]
  float4* rec;     // ((float)com64, (float)M) monopole for the interaction
  float2* rc;      // (lo, hi) fp32 thresholds on |c32 - x|^2 of the filtered
                   // opening test: d2 < lo => open, d2 > hi => accept, else
                   // the exact fp64 test; leaves
                   // hold (-inf, -inf)
  float4* tf;      // internal ids: (fl32(com64 - c32) x, y, z, fl32(s^2 / th2)):
                   // the T-phase filter data (k_force.cu tfilter_prep)
  const GridInfo* grid;  // bbox of this step (filter slack)
  double th2;            // theta^2 the thresholds were built for
  double4* mom;    // (M, Mx, My, Mz) fp64 moments (build only) [A12]
  double4* rec64 = nullptr;  // NEXT-2 FP64 mode, every id: (com64, M) of an
                             // internal node, the sorted body (x, m) at a leaf
  double4* blo64 = nullptr;  // NEXT-2 FP64 mode: fp64 AABB (build only)
  double4* bhi64 = nullptr;
  float4* blo;     // AABB lo (x, y, z, -)
  float4* bhi;     // AABB hi (x, y, z, -)
  bool quad;       // NEXT-4: build second moments, add quadrupole terms
  Quad64* S64;     // per internal node (quad only)
  float4* qf;      // per internal node, 2 x float4: (Sxx, Syy, Szz, trS), (Sxy, Sxz, Syz, 0)
};

constexpr int kMaxPeers = 8;                 // one NVSwitch domain of an HGX B200
constexpr int kBarrierSlots = 2;             // 0: state consumed, 1: state delivered
// Every rank's state buffers, barrier flags and group costs, mapped into this
// process (CUDA IPC over NVLink/NVSwitch, or plain pointers for contexts
// sharing one device).  Index = rank; the own rank's entries are local.
struct PeerTable {
  float4* pm[kMaxPeers];
  float4* vi[kMaxPeers];
  unsigned* flags[kMaxPeers];                // [kBarrierSlots][kMaxPeers] epochs per rank
  uint32_t* gcost[kMaxPeers];                // per 32-slot group: interactions of the last pass (NEXT-3(i))
  int G = 0, rank = 0;
};

struct ForceParams {
  TreeView t;
  const float4* leaves;   // sorted (x, y, z, m)
  const GridInfo* grid;   // this step's bbox (for the fp32 filter slack)
  int64_t t_begin;        // owned target slots [t_begin, t_end)
  int64_t t_end;
  double th2;             // theta^2 (fp64, used by the opening test)
  float eps2;             // eps^2 (fp32 interaction)
  double eps2_64 = 0.0;   // eps^2 (fp64 interaction, NEXT-2 FP64 mode)
  float4* acc;            // per owned slot (ax, ay, az, 0), indexed slot - t_begin
  // NEXT-2 FP64 mode (t.rec64 set): targets from leaves64, results to acc64
  const double4* leaves64 = nullptr;
  double4* acc64 = nullptr;
  uint32_t* count;        // interactions per owned slot
  unsigned long long* total;  // sum of interactions (integer atomics only)
  // NEXT-3(i) cost-weighted ranges: when part != null the owned range is
  // [part[part_rank], part[part_rank + 1]) read on the device (t_begin/t_end
  // ignored; the grid covers cap slots) and every warp stores its group's
  // interaction count into gcost of every rank in xp.
  const int64_t* part = nullptr;
  int part_rank = 0;
  int64_t cap = 0;
  PeerTable xp{};
  // Super-group pre-pass (k_force.cu K6a): per super-group of kSG
  // consecutive owned targets, the nodes every one of them accepts (acc) and
  // the frontier of nodes its box does not decide (fr); cnt = (n_acc, n_fr)
  // (the lists are bounded, never dropped; sg_cnt = null: no lists, the warps
  // start from the root).
  uint32_t* sg_acc = nullptr;
  uint32_t* sg_fr = nullptr;
  int2* sg_cnt = nullptr;
};

// Super-group size and list capacities of K6a (k_force.cu): 4096 accepted +
// 2048 frontier ids per 256 targets (96 B per body).  Lists that would
// overflow are cut short (the rest becomes frontier), never dropped; the
// round-2 lists of 2048 + 1024 overflowed on 6 % of the clustered 10^8
// super-groups and on nearly all at theta = 0.3 (profiles/r02_ab_k6.md).
#ifndef NBODY_SG
#define NBODY_SG 256
#endif
#ifndef NBODY_SG_ACC
#define NBODY_SG_ACC 4096
#endif
#ifndef NBODY_SG_FR
#define NBODY_SG_FR 2048
#endif
constexpr int kSG = NBODY_SG, kSGAcc = NBODY_SG_ACC, kSGFr = NBODY_SG_FR;
// multi-GPU partition unit [A21]: rank ranges start at multiples of it, so
// they start at super-group boundaries (256 slots, or kSG if larger)
constexpr int kPartUnitSlots = kSG > 256 ? kSG : 256;
inline int64_t sg_groups(int64_t n) { return kSG > 0 ? (n + kSG - 1) / kSG + 1 : 0; }

// ---- K1 / K2 --------------------------------------------------------------
void launch_bbox_partial(const float4* pm, int64_t n, float* partial, int nblocks, cudaStream_t s);
void launch_bbox_final(const float* partial, int nparts, int b, GridInfo* g, cudaStream_t s);
// keys + the sort's digit histograms (ghist[passes][256], must be zeroed)
void launch_keys32(const float4* pm, int64_t n, const GridInfo* g, uint32_t* keys, uint32_t* ghist, int passes,
                   cudaStream_t s);
void launch_keys64(const float4* pm, int64_t n, const GridInfo* g, unsigned long long* keys, uint32_t* ghist,
                   int passes, int b, cudaStream_t s);
// NEXT-2 FP64 mode: the same stages on fp64 bodies (x, y, z, m) as double4;
// partial[block][6] doubles; the grid's lo64/hi64 hold the box.
void launch_bbox_partial_f64(const double4* pm, int64_t n, double* partial, int nblocks, cudaStream_t s);
void launch_bbox_final_f64(const double* partial, int nparts, int b, GridInfo* g, cudaStream_t s);
void launch_keys_f64(const double4* pm, int64_t n, const GridInfo* g, void* keys, int key_bytes, uint32_t* ghist,
                     int passes, cudaStream_t s);

// ---- K3 radix sort ---------------------------------------------------------
struct SortPlan {
  int64_t n;
  int key_bytes;      // 4 or 8
  int passes;         // ceil(3b / 8)
  int64_t tiles;      // per pass
  uint32_t* ghist;    // [8][256]
  uint32_t* status;   // [passes][tiles][256]
  uint32_t* tile_ctr; // [8]
  uint32_t* gpre;     // [8][256] exclusive prefix of ghist per pass (k_hist_prefix)
  bool hist_ready;    // ghist already filled (by the key kernel)
};
int64_t sort_tiles(int64_t n);
size_t sort_scratch_bytes(int64_t n);
// Sorts (keys[0], implicit iota) into perm; keys/idx double buffers are
// clobbered.  Returns the buffer index (0/1) of idx holding the permutation.
int launch_radix_sort(const SortPlan& p, void* keys[2], uint32_t* idx[2], cudaStream_t s);

// ---- K4 / K5 ---------------------------------------------------------------
void launch_permute(const float4* pm_in, const float4* vi_in, const uint32_t* perm, int64_t n, float4* pm_out,
                    float4* vi_out, cudaStream_t s);
void launch_build(const TreeView& t, const float4* leaves, cudaStream_t s);  // level by level (reference)
// levels 1..10 fused per 1024-leaf subtree + one block for the top levels;
// keep_all also stores every node's moments/box (debug views)
int build_fused_kernels(const TreeView& t);  // kernel launches of launch_build_fused
void launch_build_fused(const TreeView& t, const float4* leaves, bool keep_all, cudaStream_t s);
// NEXT-2 FP64 mode: leaves are t.rec64 + 2^L (fp64 bodies); boxes in fp64
void launch_permute_f64(const double4* pm_in, const double4* vi_in, const uint32_t* perm, int64_t n,
                        double4* pm_out, double4* vi_out, cudaStream_t s);
void launch_build_fused_f64(const TreeView& t, bool keep_all, cudaStream_t s);

// ---- K6 --------------------------------------------------------------------
void launch_force(const ForceParams& p, int variant, cudaStream_t s);
// K6a: the super-group lists of p (p.sg_* must be set); variant-0 K6 reads them.
void launch_force_sgroups(const ForceParams& p, cudaStream_t s);
// K6 event counters (NBODY_K6_STATS builds; else returns 0); reading resets them
constexpr int kK6Stats = 52;
int force_stats(unsigned long long* out, int n, bool reset = true);

// ---- NEXT-1: all-pairs direct sum for sampled targets (fp64) ----------------
// Lazy module loading (the CUDA 12 default) loads a kernel at its first
// launch, and the loader can wait for the device to go idle; a context whose
// device barrier spins on another context of the same process (the fused
// peer exchange with graphs off) would then deadlock.  preload_*() touch
// every kernel once (cudaFuncGetAttributes), called at nbody_create.
template <class F>
inline void touch(F* f) {
  cudaFuncAttributes a;
  if (cudaFuncGetAttributes(&a, f) != cudaSuccess) cudaGetLastError();
}
void preload_allpairs();
void preload_bbox_keys();
void preload_build();
void preload_direct();
void preload_exchange();
void preload_force();
void preload_update();
void preload_sort();
// NEXT-1 fp32 all-pairs (k_allpairs.cu); target slots of ids (k_direct.cu)
void launch_target_slots(const float4* vi, int64_t n, const int64_t* ids, int64_t nt, uint32_t* slot_of,
                         uint32_t* tslot, cudaStream_t s);
int64_t allpairs_chunks(int64_t n, int64_t nt, int nsm);
void launch_allpairs32(const float4* pm, int64_t n, const uint32_t* tslot, int64_t nt, float eps2, int64_t chunks,
                       double4* part, double* out, cudaEvent_t ev0, cudaEvent_t ev1, cudaStream_t s);
int64_t direct_chunks(int64_t n, int64_t nt);
void launch_direct(const float4* pm, const float4* vi, int64_t n, const int64_t* ids, int64_t nt, double eps2,
                   uint32_t* slot_of, uint32_t* tslot, double4* part, double* out, cudaStream_t s);

// ---- K7 and helpers --------------------------------------------------------
void launch_leapfrog(const float4* pm_in, const float4* vi_in, const float4* acc, int64_t n, float dt, float4* pm_out,
                     float4* vi_out, cudaStream_t s);
void launch_fill_float2(float2* p, int64_t count, float2 v, cudaStream_t s);
// K7 with the next pass's S1 partials fused (partial[6 * nparts], nparts blocks)
void launch_leapfrog_bbox(const float4* pm_in, const float4* vi_in, const float4* acc, int64_t n, float dt,
                          float4* pm_out, float4* vi_out, float* partial, int nparts, cudaStream_t s);
void launch_pack_bodies(const float* pos, const float* vel, const float* mass, int64_t n, float4* pm, float4* vi,
                        int* bad, cudaStream_t s);
// nbody_set_state: validate a restored state (flags as k_pack, 4 = ids not a
// permutation of [0, n); seen[n] zeroed by the caller)
void launch_check_state(const float4* pm, const float4* vi, int64_t n, uint32_t* seen, int* bad, cudaStream_t s);
void launch_check_state_f64(const double4* pm, const double4* vi, int64_t n, uint32_t* seen, int* bad,
                            cudaStream_t s);
// out[id][3] <- src[slot].xyz for slots [0, n); id from vi[slot].w
void launch_scatter_by_id3(const float4* src, const float4* vi, int64_t n, float* out, cudaStream_t s);
void launch_scatter_by_id1(const uint32_t* src, const float4* vi, int64_t n, uint32_t* out, cudaStream_t s);
// NEXT-2 FP64 mode helpers: ids are vi.w (exact integers in fp64)
void launch_leapfrog_f64(const double4* pm_in, const double4* vi_in, const double4* acc, int64_t n, double dt,
                         double4* pm_out, double4* vi_out, cudaStream_t s);
void launch_pack_bodies_f64(const double* pos, const double* vel, const double* mass, int64_t n, double4* pm,
                            double4* vi, int* bad, cudaStream_t s);
void launch_scatter_by_id3_f64(const double4* src, const double4* vi, int64_t n, double* out, cudaStream_t s);
void launch_scatter_by_id3_f64to32(const double4* src, const double4* vi, int64_t n, float* out, cudaStream_t s);
void launch_scatter_by_id1_f64(const uint32_t* src, const double4* vi, int64_t n, uint32_t* out, cudaStream_t s);

// ---- K7 fused with the exchange over peer memory -------------
// Leapfrog of the owned slots [b, b + len) (acc indexed from 0), storing the
// new records straight into slot b + i of EVERY rank's pm0/vi0.
// With part != null the range is [part[rank], part[rank + 1]) read on the
// device and len is only the launch bound (cap).
void launch_leapfrog_scatter(const float4* pm_in, const float4* vi_in, const float4* acc, int64_t b, int64_t len,
                             float dt, const PeerTable& pt, const int64_t* part, cudaStream_t s);
// NEXT-3(i): next step's cost-weighted ranges from the 32-slot group costs
// of the last pass (identical on every rank): part[0..G] <- boundaries
// (multiples of 256 slots [A21], each slice <= cap_units units of 256);
// used[0..G] <- the old part.
void launch_partition(const uint32_t* gcost, int64_t groups, int G, int64_t n, int64_t cap_units, int64_t* part,
                      int64_t* used, cudaStream_t s);
// Device-side barrier over the G ranks: signal epoch+1 of `slot` to every
// rank (release, system scope), then wait until every rank's signal for
// that epoch arrived in the own flag block (acquire).  A wait longer than
// ~20 s sets *err and returns.
void launch_xbarrier(const PeerTable& pt, unsigned* epoch, int slot, int* err, cudaStream_t s);

}  // namespace nb
