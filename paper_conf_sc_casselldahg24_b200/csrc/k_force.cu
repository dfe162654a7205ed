// K6 CALCULATEFORCE over the Hilbert-sorted BVH (
// Eq. 1 P:72 with Plummer softening [A1], G = 1 [A2]).
//
// Semantics (identical to the oracle's per-body DFS): for target k, node n
// is in k's interaction list iff every proper ancestor of n fails the
// opening test for k and n passes it (or n is a leaf other than k).  The
// opening test is the fixed fp64 expression [A3][A16][A20]
//     s^2 < theta^2 * fma(dz, dz, fma(dy, dy, dx*dx)),  d = com64 - x_k,
// so every decision -- hence every interaction list -- is bit-identical to
// the oracle's.  The interaction itself is fp32 (MUFU rsqrt + FMA) on the
// monopole ((float)com, (float)M); its summation order is free
// (tolerance-checked).  Interactions with r == 0 (the target itself, or a
// coincident body when eps == 0) add exactly 0.
//
// Tree addressing: heap ids (capi.cu plan_tree): root 1, children of g are
// 2g and 2g+1, leaf i is 2^L + i, level of g is L - floor(log2 g).  rec[g]
// is the fp32 monopole (the sorted body for a leaf), rc[g] the fp32 filter
// thresholds on the squared distance, pred[g] the exact fp64 (com, s^2) of
// an internal node.
//
// Variant 0 (default), group-classified transposed walk.  A warp owns 32
// Hilbert-consecutive targets with bounding box B.
//   K6a (k_force_sgroups, a separate kernel launched first): one warp per
//      super-group of kSG = 256 consecutive targets runs the box phase below
//      against the super-group's box from the root; the nodes every target
//      of the super-group accepts go to its `acc` list, the nodes it cannot
//      decide (and leaves) to its `frontier`.  A variant-0 warp appends `acc`
//      as full dense entries and starts its own box phase from the frontier
//      instead of the root (same lists: its box lies inside the super-group's).
//   A. Box phase (lanes = nodes): lanes classify 32 nodes at a time against B
//      with exact fp64 bounds of the opening test over all of B: every lane
//      accepts (-> dense list, all lanes), every lane opens (-> children are
//      box-classified next) or mixed (-> T with all lanes in the mask).
//      Every node reaching A has been opened by every lane, so this is exact.
//   T. Transposed phase (lanes = nodes, loop over targets): each lane takes a
//      (node, mask of the targets that reached it) entry and evaluates the
//      per-target opening test for all 32 targets, whose positions are
//      broadcast from shared memory -- one warp instruction decides 32
//      node-target pairs.  Accepting targets -> a dense entry (record, mask);
//      opening targets -> both children enter T with that mask.  Leaves carry
//      thresholds (-inf, -inf): always accepted, except by the target itself.
//   D. Dense phase (lanes = targets): each entry is read once from shared
//      memory (broadcast) and every lane in its mask interacts with it; full-
//      mask and partial-mask entries are kept in separate lists.
// Variant 1, the mask-stack walk from the root for every warp (the simpler
// exact design, kept as a cross-check and as the overflow path of T).
//
// Mask stack: a warp-uniform DFS stack of (sibling pair, mask of the lanes
// that reached it), held in registers (lane i holds entry i; depth <= L+1 <
// 32).  Each popped pair is loaded once for the warp (one 32-byte load),
// lanes in the mask test both siblings, accepting lanes interact, and the
// ballots of opening lanes become the masks of the children pairs.  No lane
// ever visits a node outside its own DFS, so lists are exact.
//
// Per-lane opening decisions use an fp32 filter with a rigorous error bound
// and fall back to the exact fp64 expression inside the uncertainty band
// (DESIGN.md "fp32 filter"), so they equal the fp64 decisions.
#include <type_traits>

#include "internal.cuh"

// Design/debug build (-DNBODY_DEBUG_BOUNDS): device-side bounds checks on
// every list and stack write of K6 and K6a (a failed check traps the kernel);
// the stand-in for compute-sanitizer memcheck, which the GPU pool no longer
// offers (tests/test_small_caps_gpu.py runs the tiny-capacity builds with it).
#ifdef NBODY_DEBUG_BOUNDS
#include <cstdio>
#define NB_CHECK(cond)                                                                              \
  do {                                                                                              \
    if (!(cond)) {                                                                                  \
      printf("NB_CHECK failed: %s (%s:%d)\n", #cond, __FILE__, __LINE__);                            \
      __trap();                                                                                     \
    }                                                                                               \
  } while (0)
#else
#define NB_CHECK(cond) ((void)0)
#endif

namespace nb {

// Traversal event counters for design work (NBODY_K6_STATS builds only;
// read with nbody_debug_force_stats).  Index meaning: see kStatNames in
// scripts/k6_stats.py.
#ifdef NBODY_K6_STATS
__device__ unsigned long long g_k6_stats[kK6Stats];
#define K6STAT(i, v) (st[i] += (v))
#else
#define K6STAT(i, v) ((void)0)
#endif

int force_stats(unsigned long long* out, int n, bool reset) {
#ifdef NBODY_K6_STATS
  if (n > kK6Stats) n = kK6Stats;
  if (cudaMemcpyFromSymbol(out, g_k6_stats, sizeof(unsigned long long) * n) != cudaSuccess) return -1;
  static const unsigned long long zero[kK6Stats] = {};
  if (reset && cudaMemcpyToSymbol(g_k6_stats, zero, sizeof(zero)) != cudaSuccess) return -1;
  return n;
#else
  (void)reset;
  (void)out;
  (void)n;
  return 0;
#endif
}

namespace {

constexpr unsigned kFull = 0xffffffffu;

__device__ __forceinline__ float rsqrt_fast(float x) {
  float y;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// One 32-byte load of a sibling pair of records (g even => 32-B aligned).
__device__ __forceinline__ void load_pair(const float4* p, float4& a, float4& b) {
  asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w)
               : "l"(p));
}

// Exact fp64 opening test (the definition).
__device__ __forceinline__ bool opening_accept64(const double4& p, double x, double y, double z, double th2) {
  const double dx = __dsub_rn(p.x, x);
  const double dy = __dsub_rn(p.y, y);
  const double dz = __dsub_rn(p.z, z);
  const double d2 = __fma_rn(dz, dz, __fma_rn(dy, dy, __dmul_rn(dx, dx)));
  return p.w < __dmul_rn(th2, d2);
}

struct Target {
  float x, y, z;    // the lane's target position (fp32; rounded in FP64 mode)
  float eps2;
  double th2;
  double x64 = 0.0, y64 = 0.0, z64 = 0.0;  // NEXT-2 FP64 mode: the exact position
  double eps2_64 = 0.0;
};

struct Acc {
  float x = 0.f, y = 0.f, z = 0.f;
  uint32_t n = 0;
  // add m r / (|r|^2 + eps^2)^(3/2) when `on`; d2 = |r|^2 already computed
  __device__ __forceinline__ void add(bool on, float dx, float dy, float dz, float d2, float m, float eps2) {
    const float r2 = d2 + eps2;
    const float inv = r2 > 0.f ? rsqrt_fast(r2) : 0.f;
    const float w = on ? m * inv * inv * inv : 0.f;
    x = fmaf(w, dx, x);
    y = fmaf(w, dy, y);
    z = fmaf(w, dz, z);
  }
};

// NEXT-2 FP64 mode accumulator and interaction (the paper's precision,
// P:272): a += m r / (|r|^2 + eps^2)^(3/2), r = s - x, all in fp64; r2 == 0
// (eps = 0, coincident) adds exactly 0 [A1].
struct AccD {
  double x = 0.0, y = 0.0, z = 0.0;
  uint32_t n = 0;
};

template <bool kSoft>
__device__ __forceinline__ void interact64(AccD& a, const double4& s, double m, const Target& T) {
  const double dx = s.x - T.x64, dy = s.y - T.y64, dz = s.z - T.z64;
  const double r2 = fma(dz, dz, fma(dy, dy, fma(dx, dx, T.eps2_64)));
  double inv = rsqrt(r2);
  if (!kSoft) inv = r2 > 0.0 ? inv : 0.0;
  const double w = (m * inv) * (inv * inv);
  a.x = fma(w, dx, a.x);
  a.y = fma(w, dy, a.y);
  a.z = fma(w, dz, a.z);
}

// NEXT-4 [A24]: the quadrupole term of internal node qid (the oracle's
// interact_quad in fp32): with d = com - x, inv = (|d|^2 + eps^2)^(-1/2),
//   a += [(15/2) d.S.d inv^7 - (3/2) tr(S) inv^5] d - 3 (S d) inv^5.
// qf[2 qid] = (Sxx, Syy, Szz, trS), qf[2 qid + 1] = (Sxy, Sxz, Syz, 0).
__device__ __forceinline__ void quad_term(Acc& a, float dx, float dy, float dz, float inv,
                                          const float4* __restrict__ qf, uint32_t qid, bool on) {
  const float4 q0 = __ldg(qf + 2 * size_t(qid)), q1 = __ldg(qf + 2 * size_t(qid) + 1);
  const float inv2 = inv * inv;
  const float inv5 = inv2 * inv2 * inv;
  const float inv7 = inv5 * inv2;
  const float sx = fmaf(q0.x, dx, fmaf(q1.x, dy, q1.y * dz));
  const float sy = fmaf(q1.x, dx, fmaf(q0.y, dy, q1.z * dz));
  const float sz = fmaf(q1.y, dx, fmaf(q1.z, dy, q0.z * dz));
  const float dsd = fmaf(dx, sx, fmaf(dy, sy, dz * sz));
  const float c = on ? fmaf(7.5f * dsd, inv7, -1.5f * q0.w * inv5) : 0.f;
  const float e = on ? -3.f * inv5 : 0.f;
  a.x = fmaf(c, dx, fmaf(e, sx, a.x));
  a.y = fmaf(c, dy, fmaf(e, sy, a.y));
  a.z = fmaf(c, dz, fmaf(e, sz, a.z));
}

struct Probe {
  float dx, dy, dz, d2;
};

__device__ __forceinline__ Probe probe(const float4& r, const Target& T) {
  Probe p;
  p.dx = r.x - T.x;
  p.dy = r.y - T.y;
  p.dz = r.z - T.z;
  p.d2 = fmaf(p.dz, p.dz, fmaf(p.dy, p.dy, p.dx * p.dx));
  return p;
}

// Loop invariants of the walk, pinned in registers.
struct Walk {
  const float4* rec;
  const float4* rc2;     // rc viewed as pairs (lo_A, hi_A, lo_B, hi_B)
  const float2* rc;
  const double4* pred;
  const double4* rec64;  // NEXT-2 FP64 mode records (or null)
  const float4* qf;      // NEXT-4 quadrupoles (2 float4 per id) or null
  uint32_t leaf0, n;
  int L;
};

template <class T>
__device__ __forceinline__ T* in_reg(T* p) {
  asm volatile("" : "+l"(p));
  return p;
}

__device__ __forceinline__ Walk make_walk(const ForceParams& P) {
  Walk W;
  W.rec = in_reg(P.t.rec);
  W.rc = in_reg(P.t.rc);
  W.rc2 = reinterpret_cast<const float4*>(W.rc);
  W.pred = in_reg(P.t.pred);
  W.rec64 = P.t.rec64;
  W.qf = P.t.qf;
  W.L = P.t.L;
  W.leaf0 = 1u << W.L;
  W.n = uint32_t(P.t.n);
  return W;
}

// Per-lane decision for one internal node: fp32 filter, fp64 fallback.
__device__ __forceinline__ bool decide1(const Walk& W, uint32_t g, bool in, float d2, float2 c, const Target& T) {
  bool acc = in && d2 > c.y;
  const bool und = in && !acc && !(d2 < c.x);
  if (__any_sync(kFull, und)) {
    if (und) acc = W.rec64 ? opening_accept64(W.pred[g], T.x64, T.y64, T.z64, T.th2)
                           : opening_accept64(W.pred[g], T.x, T.y, T.z, T.th2);
  }
  return acc;
}

// One mask-walk interaction with record r (fp32) / node id g (FP64 mode:
// the fp64 record rec64[g]).
__device__ __forceinline__ void walk_add(Acc& a, bool on, const Probe& p, const float4& r, const Walk&, uint32_t,
                                         const Target& T) {
  a.add(on, p.dx, p.dy, p.dz, p.d2, r.w, T.eps2);
}
__device__ __forceinline__ void walk_add(AccD& a, bool on, const Probe&, const float4&, const Walk& W, uint32_t g,
                                         const Target& T) {
  if (on) {
    const double4 s = W.rec64[g];
    interact64<false>(a, s, s.w, T);
  }
}

// The per-lane mask-stack walk of the subtree of node g0 for the lanes in
// mask0 (all of which reached g0).
// NEXT-4: quadrupole of an accepted internal node in the mask walk.
__device__ __forceinline__ void quad_at(Acc& a, const Probe& p, float eps2, const float4* qf, uint32_t g, bool on) {
  const float r2 = p.d2 + eps2;
  const float inv = r2 > 0.f ? rsqrt_fast(r2) : 0.f;
  quad_term(a, p.dx, p.dy, p.dz, inv, qf, g, on);
}

template <bool kQuad, class AccT>
__device__ __forceinline__ void mask_walk(const Walk& W, const Target& T, uint32_t kid, AccT& a, int lane, uint32_t g0,
                                          uint32_t mask0) {
  // the start node on its own
  {
    const bool in = (mask0 >> lane) & 1u;
    const float4 r = __ldg(W.rec + g0);
    const Probe p = probe(r, T);
    if (g0 >= W.leaf0) {  // a leaf (N == 1 root)
      const bool acc = in && g0 != kid;
      walk_add(a, acc, p, r, W, g0, T);
      a.n += acc;
      return;
    }
    const bool acc = decide1(W, g0, in, p.d2, __ldg(W.rc + g0), T);
    if (__any_sync(kFull, acc)) {
      walk_add(a, acc, p, r, W, g0, T);
      if constexpr (kQuad) quad_at(a, p, T.eps2, W.qf, g0, acc);
    }
    a.n += acc;
    const uint32_t rej = __ballot_sync(kFull, in && !acc);
    if (rej == 0) return;
    mask0 = rej;
    g0 = 2u * g0;
  }
  // sibling pairs; lane i holds stack entry i (depth <= L + 1 < 32)
  uint32_t sg = g0, sm = mask0;
  int sp = 1;
  while (sp > 0) {
    --sp;
    const uint32_t g = __shfl_sync(kFull, sg, sp);
    const uint32_t em = __shfl_sync(kFull, sm, sp);
    const int l = W.L - 31 + __clz(int(g));
    const bool in = (em >> lane) & 1u;
    const bool hasB = (((g + 1u) << l) - W.leaf0) < W.n;  // right sibling exists iff its first leaf < N
    float4 rA, rB;
    load_pair(W.rec + g, rA, rB);
    const Probe pA = probe(rA, T);
    const Probe pB = probe(rB, T);
    bool accA, accB;
    if (l == 0) {  // leaves: exact interactions, the target itself excluded
      accA = in && g != kid;
      accB = in && hasB && g + 1u != kid;
    } else {
      const float4 c = __ldg(W.rc2 + (g >> 1));
      accA = in && pA.d2 > c.y;
      accB = in && hasB && pB.d2 > c.w;
      const bool undA = in && !accA && !(pA.d2 < c.x);
      const bool undB = in && hasB && !accB && !(pB.d2 < c.z);
      if (__any_sync(kFull, undA || undB)) {  // rare: exact fp64 decision
        const double ex = W.rec64 ? T.x64 : double(T.x), ey = W.rec64 ? T.y64 : double(T.y),
                     ez = W.rec64 ? T.z64 : double(T.z);
        if (undA) accA = opening_accept64(W.pred[g], ex, ey, ez, T.th2);
        if (undB) accB = opening_accept64(W.pred[g + 1], ex, ey, ez, T.th2);
      }
      const uint32_t rejB = __ballot_sync(kFull, in && hasB && !accB);
      const uint32_t rejA = __ballot_sync(kFull, in && !accA);
      // push the children pair of B, then of A (A's subtree is walked first)
      const bool pushB = rejB != 0, pushA = rejA != 0;
      if (pushB && lane == sp) { sg = 2u * g + 2u; sm = rejB; }
      const int q = sp + int(pushB);
      if (pushA && lane == q) { sg = 2u * g; sm = rejA; }
      sp = q + int(pushA);
    }
    if (__any_sync(kFull, accA)) {
      walk_add(a, accA, pA, rA, W, g, T);
      if constexpr (kQuad) { if (l > 0) quad_at(a, pA, T.eps2, W.qf, g, accA); }
    }
    if (__any_sync(kFull, accB)) {
      walk_add(a, accB, pB, rB, W, g + 1u, T);
      if constexpr (kQuad) { if (l > 0) quad_at(a, pB, T.eps2, W.qf, g + 1u, accB); }
    }
    a.n += accA;
    a.n += accB;
  }
}

template <bool kF64 = false>
__device__ __forceinline__ Target load_target(const ForceParams& P, int64_t k, bool active) {
  Target T;
  if constexpr (kF64) {  // NEXT-2: exact fp64 target, fp32 rounding for the filters
    const double4 me = active ? P.leaves64[k] : make_double4(0.0, 0.0, 0.0, 0.0);
    T.x64 = me.x;
    T.y64 = me.y;
    T.z64 = me.z;
    T.x = float(me.x);
    T.y = float(me.y);
    T.z = float(me.z);
    T.eps2_64 = P.eps2_64;
  } else {
    const float4 me = active ? P.leaves[k] : make_float4(0.f, 0.f, 0.f, 0.f);
    T.x = me.x;
    T.y = me.y;
    T.z = me.z;
  }
  T.th2 = P.th2;
  T.eps2 = P.eps2;
  return T;
}

// The owned target range: static, or (NEXT-3(i)) read from the device.
__device__ __forceinline__ void owned_range(const ForceParams& P, int64_t& tb, int64_t& te) {
  if (P.part) {
    tb = P.part[P.part_rank];
    te = P.part[P.part_rank + 1];
  } else {
    tb = P.t_begin;
    te = P.t_end;
  }
}

// k: this lane's slot; k0: the warp's first slot (a multiple of 32 from 0).
template <class AccT>
__device__ __forceinline__ void store_result(const ForceParams& P, int64_t tb, int64_t k, int64_t k0, bool active,
                                             const AccT& a, int lane) {
  if (active) {
    if constexpr (sizeof(a.x) == 8)
      P.acc64[k - tb] = make_double4(a.x, a.y, a.z, 0.0);
    else
      P.acc[k - tb] = make_float4(a.x, a.y, a.z, 0.f);
    P.count[k - tb] = a.n;
  }
  const uint32_t tot = __reduce_add_sync(kFull, active ? a.n : 0u);
  if (lane == 0) {
    atomicAdd(P.total, (unsigned long long)tot);
    if (P.part)  // NEXT-3(i): this group's cost, to every rank
      for (int q = 0; q < P.xp.G; ++q) P.xp.gcost[q][k0 >> 5] = tot;
  }
}

// The same for variant 0, from 32-bit quantities that stay live anyway:
// idx = k - tb (this lane's owned index), k0u = the warp's first slot.
template <class AccT>
__device__ __forceinline__ void store_result_idx(const ForceParams& P, uint32_t idx, uint32_t k0u, bool active,
                                                 const AccT& a, int lane) {
  if (active) {
    if constexpr (sizeof(a.x) == 8)
      P.acc64[idx] = make_double4(a.x, a.y, a.z, 0.0);
    else
      P.acc[idx] = make_float4(a.x, a.y, a.z, 0.f);
    P.count[idx] = a.n;
  }
  const uint32_t tot = __reduce_add_sync(kFull, active ? a.n : 0u);
  if (lane == 0) {
    atomicAdd(P.total, (unsigned long long)tot);
    if (P.part)  // NEXT-3(i): this group's cost, to every rank
      for (int q = 0; q < P.xp.G; ++q) P.xp.gcost[q][k0u >> 5] = tot;
  }
}

// ------------------------------------------------------------ variant 1 ----
constexpr int kV1Warps = 8;

template <bool kQuad>
__global__ __launch_bounds__(32 * kV1Warps) void k_force_maskstack(const ForceParams P) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int64_t tb, te;
  owned_range(P, tb, te);
  const int64_t k0 = tb + (int64_t(blockIdx.x) * kV1Warps + w) * 32;
  const int64_t k = k0 + lane;
  const bool active = k < te;
  const uint32_t amask = __ballot_sync(kFull, active);
  if (amask == 0) return;
  const Target T = load_target(P, k, active);
  Acc a;
  const Walk W = make_walk(P);
  const uint32_t kid = W.leaf0 + uint32_t(k);
  mask_walk<kQuad>(W, T, kid, a, lane, 1u, amask);
  store_result(P, tb, k, k0, active, a, lane);
}


// ------------------------------------------------------------ variant 2 ----
// The paper's own CALCULATEFORCE scheme, for comparison: one thread per
// target body walking the BVH depth-first without a stack by the skip-list
// jumps of P:222 / P:245 [A7] -- cursor (l, s) = the node of level l whose
// first leaf is s; open: l <- l - 1; done with a node: s <- s + 2^l, stop at
// s >= N, else l <- min(ctz(s), L).  The decisions are the same fp32-filtered
// fp64 test per lane (no warp votes: lanes diverge freely), so the lists --
// and the counts -- equal the other variants'.  Monopole only.
constexpr int kV2Threads = 256;

__global__ __launch_bounds__(kV2Threads) void k_force_skiplist(const ForceParams P) {
  const int lane = threadIdx.x & 31;
  int64_t tb, te;
  owned_range(P, tb, te);
  const int64_t k0 = tb + int64_t(blockIdx.x) * kV2Threads + (threadIdx.x & ~31);
  const int64_t k = k0 + lane;
  const bool active = k < te;
  // idle warps past the range end store nothing (their gcost entry belongs
  // to the next rank, or lies past the last group)
  if (__ballot_sync(kFull, active) == 0) return;
  const Target T = load_target(P, k, active);
  const Walk W = make_walk(P);
  const uint32_t kid = W.leaf0 + uint32_t(k);
  Acc a;
  int l = W.L;
  uint32_t sl = 0;  // first leaf of the current node
  while (active) {
    const uint32_t g = (W.leaf0 + sl) >> l;
    const float4 r = __ldg(W.rec + g);
    const Probe pr = probe(r, T);
    bool take;  // interact with this node and skip its subtree
    if (l == 0) {
      take = true;
      const bool on = g != kid;  // a leaf never acts on itself
      a.add(on, pr.dx, pr.dy, pr.dz, pr.d2, r.w, T.eps2);
      a.n += on;
    } else {
      const float2 c = __ldg(W.rc + g);
      take = pr.d2 > c.y;
      if (!take && !(pr.d2 < c.x)) take = opening_accept64(W.pred[g], T.x, T.y, T.z, T.th2);
      if (take) {
        a.add(true, pr.dx, pr.dy, pr.dz, pr.d2, r.w, T.eps2);
        ++a.n;
      }
    }
    if (take) {
      sl += 1u << l;
      if (sl >= W.n) break;
      l = min(__ffs(int(sl)) - 1, W.L);
    } else {
      --l;
    }
  }
  store_result(P, tb, k, k0, active, a, lane);
}

// ------------------------------------------------------------ variant 0 ----
#ifndef NBODY_V0_WARPS
#define NBODY_V0_WARPS 4
#endif
constexpr int kV0Warps = NBODY_V0_WARPS;
// Sized for 6 blocks x 4 warps per SM: 80 registers per thread and 31 KB of
// shared memory per block (round 2: 6 blocks with these lists beat 8 blocks
// at 64 registers by 3.7 %, profiles/r02_ab_k6.md); stack overflow is
// handled (box phase: hand over as MIXED; transposed phase: per-lane mask
// walk; K6a frontier: refilled in chunks), so the capacities only affect speed.
#ifndef NBODY_CAP_T
#define NBODY_CAP_T 256
#endif
#ifndef NBODY_V0_MINB
#define NBODY_V0_MINB 6
#endif
#ifndef NBODY_SMEM_TOP
#define NBODY_SMEM_TOP 0
#endif

#ifndef NBODY_CAP_A
#define NBODY_CAP_A 320
#endif
constexpr int kCapA = NBODY_CAP_A;  // box-phase stack (ids)
constexpr int kCapT = NBODY_CAP_T;  // transposed-phase stack (id, mask)
#ifndef NBODY_CAP_F
#define NBODY_CAP_F 96
#endif
#ifndef NBODY_CAP_P
#define NBODY_CAP_P 96
#endif
#ifndef NBODY_FUNROLL
#define NBODY_FUNROLL 2
#endif
#ifndef NBODY_PUNROLL
#define NBODY_PUNROLL 2
#endif
constexpr int kFUnroll = NBODY_FUNROLL, kPUnroll = NBODY_PUNROLL;  // dense loop unrolling (#pragma takes no macros)
#ifndef NBODY_LEAF_DIRECT
#define NBODY_LEAF_DIRECT 1
#endif
constexpr int kCapF = NBODY_CAP_F;  // dense list: entries every active lane interacts with
constexpr int kCapP = NBODY_CAP_P;  // dense list: entries with a lane mask
// NEXT-4 quadrupole variant: the staged second moments (32 B per entry) make
// the lists larger, so the full list and the T stack are shortened to keep 5
// blocks per SM (measured: 70.3 ms at 4 blocks, 66.8 at 5, uniform 1e7).
// NEXT-2 FP64 mode (32-B fp64 records): 64 full entries, 192 T slots and at
// most 72 registers give 6 blocks per SM (disks 1e7: 67.7 ms at 4 blocks with
// 124 registers, 58.0 ms here; 128 T slots overflow too often: 75.9 ms).
#ifndef NBODY_QCAP_F
#define NBODY_QCAP_F 64
#endif
#ifndef NBODY_QCAP_T
#define NBODY_QCAP_T 224
#endif
#ifndef NBODY_QCAP_A
#define NBODY_QCAP_A 256
#endif
template <bool kQuad, bool kF64> constexpr int cap_f() { return kQuad ? NBODY_QCAP_F : kF64 ? 64 : kCapF; }
// box-phase stack: the quadrupole and FP64 variants keep a smaller one (their
// larger records leave less shared memory)
#ifndef NBODY_F64CAP_A
#define NBODY_F64CAP_A 128
#endif
template <bool kQuad, bool kF64> constexpr int cap_a() {
  return kQuad ? NBODY_QCAP_A : kF64 ? NBODY_F64CAP_A : kCapA;
}
#ifndef NBODY_QCAP_P
#define NBODY_QCAP_P 64
#endif
#ifndef NBODY_F64CAP_P
#define NBODY_F64CAP_P 64
#endif
template <bool kQuad, bool kF64> constexpr int cap_p() { return kQuad ? NBODY_QCAP_P : kF64 ? NBODY_F64CAP_P : kCapP; }
template <bool kQuad, bool kF64> constexpr int cap_t() { return kQuad ? NBODY_QCAP_T : kF64 ? 192 : kCapT; }

// Records in pairs, component-interleaved, so that one 16-B shared load
// yields (x_a, x_b, y_a, y_b) and the interaction of two entries runs on the
// packed f32x2 pipe (FADD2/FFMA2/FMUL2: half the issue slots, same rounding
// per element as the scalar instructions).
struct alignas(16) RecPair {
  float2 x, y, z, m;
  __device__ __forceinline__ void put(int h, const float4& r) {
    reinterpret_cast<float*>(&x)[h] = r.x;
    reinterpret_cast<float*>(&y)[h] = r.y;
    reinterpret_cast<float*>(&z)[h] = r.z;
    reinterpret_cast<float*>(&m)[h] = r.w;
  }
};
// NEXT-4 [A24]: the fp32 second moments of two entries, component-
// interleaved like RecPair (qf layout: (Sxx, Syy, Szz, trS), (Sxy, Sxz, Syz)).
struct alignas(16) QuadPair {
  float2 xx, yy, zz, tr, xy, xz, yz, pad;
  __device__ __forceinline__ void put(int h, const float4& q0, const float4& q1) {
    reinterpret_cast<float*>(&xx)[h] = q0.x;
    reinterpret_cast<float*>(&yy)[h] = q0.y;
    reinterpret_cast<float*>(&zz)[h] = q0.z;
    reinterpret_cast<float*>(&tr)[h] = -1.5f * q0.w;  // -(3/2) tr S, pre-scaled for the radial coefficient
    reinterpret_cast<float*>(&xy)[h] = q1.x;
    reinterpret_cast<float*>(&xz)[h] = q1.y;
    reinterpret_cast<float*>(&yz)[h] = q1.z;
  }
};
// Targets in pairs for the transposed test, relative to the group reference
// point g: p = 2 x', q = -|x'|^2 with x' = fl(x - g) (see tfilter_prep).
struct alignas(16) TgtPair {
  float2 px, py, pz, q;
};

template <bool kQuad, bool kF64_ = false>
struct alignas(16) V0Smem {
  static constexpr bool kF64 = kF64_;
  TgtPair tgt[16];          // the warp's targets for the transposed test (paired)
  float4 tpos[kF64 ? 1 : 32];   // the warp's target positions (fp64 fallback)
  double4 tpos64[kF64 ? 32 : 1];  // NEXT-2 FP64 mode: exact target positions
  static constexpr int kF = cap_f<kQuad, kF64_>(), kT = cap_t<kQuad, kF64_>();
  RecPair frec[kF64 ? 1 : kF / 2];  // monopole / body records, all lanes
  static constexpr int kP = cap_p<kQuad, kF64_>();
  RecPair prec[kF64 ? 1 : kP / 2];  // monopole / body records, ...
  double4 frec64[kF64 ? kF : 1];    // NEXT-2 FP64 mode: the same lists in fp64
  double4 prec64[kF64 ? kP : 1];
  uint32_t pmsk[kP];        // ... for the lanes in the mask
  static constexpr int kA = cap_a<kQuad, kF64_>();
  uint32_t astk[kA];
  uint2 tstk[kT];     // (id, mask of the targets that reached it)
  int sg_next, sg_nfr;  // super-group frontier: next entry, length (K6a)
  using QP = typename std::conditional<kQuad, QuadPair, char>::type;
  QP fq[kQuad ? kF / 2 : 1];  // NEXT-4: each entry's second moments (0 for a body), paired
  QP pq[kQuad ? kP / 2 : 1];
};

__device__ __forceinline__ float warp_minf(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fminf(v, __shfl_xor_sync(kFull, v, o));
  return v;
}
__device__ __forceinline__ float warp_maxf(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(kFull, v, o));
  return v;
}

__device__ __forceinline__ float2 f2(float v) { return make_float2(v, v); }
#ifdef NBODY_K6_STATS
__device__ __forceinline__ float inf_stat() { return __int_as_float(0x7f800000); }
#endif


// Transposed-phase filter of the fp64 opening test.
// With g the group reference point (fp32), c~ = com64 - g, x~ = x - g (exact
// reals): D^2 = |com64 - x|^2 = |c~|^2 - S*,  S* = 2 c~.x~ - |x~|^2.  Each
// target evaluates S = fma(2x'_x, c'_x, fma(2x'_y, c'_y, fma(2x'_z, c'_z, q)))
// in fp32 from x' = fl(x - g), q = fl(-|x'|^2) and the node's
// c' = fl(fl(c32 - g) + lo), lo = fl32(com64 - c32) (tf).  With b >= |x~|,
// R >= every |coordinate| and L1 = |c'|_1:
//   |c' - c~|_i <= 2.01u |c~_i| + 4u^2 R,  |S - S*| <= u b (12.2 L1 + 6.2 b + 24u R),
//   | fl(|c'|^2) - |c~|^2 | <= 7.1u a2 + 8u^2 R L1          (u = 2^-24),
// so with E2 = u ((13 b + 5e-7 R) L1 + 7 b^2 + 2e-6 b R) (kk1 = 13 b + 5e-7 R,
// kk0 = 7 b^2 + 2e-6 b R, per warp) and q32 = fl32(s^2/th2) (error <= 1.01u):
//   S < KA = a2 (1 - 8u) - q32 (1 + 2u) - E2  (rounded down)  =>  D^2 > q (1 + 2e-15)
//        => the fp64 test accepts;
//   S > KO = a2 (1 + 8u) - q32 (1 - 2u) + E2  (rounded up)    =>  D^2 < q (1 - 2e-15)
//        => it opens;
// otherwise (or NaN) the exact fp64 test decides.  theta = 0: q32 = +inf, so
// KA = KO = -inf (everything opens).
__device__ __forceinline__ void tfilter_prep(const float4& r, const float4& tf, float gx, float gy, float gz,
                                             float kk1, float kk0, float& cx, float& cy, float& cz, float& KA,
                                             float& KO) {
  cx = (r.x - gx) + tf.x;
  cy = (r.y - gy) + tf.y;
  cz = (r.z - gz) + tf.z;
  const float L1 = __fadd_ru(__fadd_ru(fabsf(cx), fabsf(cy)), fabsf(cz));
  const float E2 = __fmul_ru(__fmaf_ru(kk1, L1, kk0), 5.9604644775390625e-08f);
  const float a2 = fmaf(cz, cz, fmaf(cy, cy, cx * cx));
  constexpr float kU8m = 1.f - 8.f * 5.9604644775390625e-08f, kU8p = 1.f + 8.f * 5.9604644775390625e-08f;
  constexpr float kU2m = 1.f - 2.f * 5.9604644775390625e-08f, kU2p = 1.f + 2.f * 5.9604644775390625e-08f;
  KA = __fsub_rd(__fsub_rd(__fmul_rd(a2, kU8m), __fmul_ru(tf.w, kU2p)), E2);
  KO = __fadd_ru(__fsub_ru(__fmul_ru(a2, kU8p), __fmul_rd(tf.w, kU2m)), E2);
}

// Two monopole interactions on the packed pipe; same per-element operations
// and order as interact().  (ax, ay, az) hold two partial sums each.
template <bool kSoft>
__device__ __forceinline__ void interact2(float2& ax, float2& ay, float2& az, const RecPair& s, float2 m,
                                          float2 nx, float2 ny, float2 nz, float2 eps2) {
  const float2 dx = __fadd2_rn(s.x, nx), dy = __fadd2_rn(s.y, ny), dz = __fadd2_rn(s.z, nz);
  const float2 r2 = __ffma2_rn(dz, dz, __ffma2_rn(dy, dy, __ffma2_rn(dx, dx, eps2)));
  float2 inv = make_float2(rsqrt_fast(r2.x), rsqrt_fast(r2.y));
  if (!kSoft) {
    inv.x = r2.x > 0.f ? inv.x : 0.f;
    inv.y = r2.y > 0.f ? inv.y : 0.f;
  }
  const float2 w = __fmul2_rn(__fmul2_rn(m, inv), __fmul2_rn(inv, inv));  // m inv^3, two-deep
  ax = __ffma2_rn(w, dx, ax);
  ay = __ffma2_rn(w, dy, ay);
  az = __ffma2_rn(w, dz, az);
}

// Two monopole + quadrupole interactions on the packed pipe [A24]: with
// d = s - x and inv = (|d|^2 + eps^2)^(-1/2),
//   a += {m inv^3 + [(15/2) d.S.d inv^2 - (3/2) tr(S)] inv^5} d - 3 (S d) inv^5.
// `on` (per half) masks the whole term; bodies carry S = 0.
template <bool kSoft>
__device__ __forceinline__ void interact2_quad(float2& ax, float2& ay, float2& az, const RecPair& s,
                                               const QuadPair& q, bool on0, bool on1, float2 nx, float2 ny,
                                               float2 nz, float2 eps2) {
  const float2 dx = __fadd2_rn(s.x, nx), dy = __fadd2_rn(s.y, ny), dz = __fadd2_rn(s.z, nz);
  const float2 r2 = __ffma2_rn(dz, dz, __ffma2_rn(dy, dy, __ffma2_rn(dx, dx, eps2)));
  float2 inv = make_float2(rsqrt_fast(r2.x), rsqrt_fast(r2.y));
  if (!kSoft) {
    inv.x = r2.x > 0.f ? inv.x : 0.f;
    inv.y = r2.y > 0.f ? inv.y : 0.f;
  }
  const float2 inv2 = __fmul2_rn(inv, inv);
  const float2 inv3 = __fmul2_rn(inv2, inv);
  const float2 inv5 = __fmul2_rn(inv3, inv2);
  const float2 sx = __ffma2_rn(q.xx, dx, __ffma2_rn(q.xy, dy, __fmul2_rn(q.xz, dz)));
  const float2 sy = __ffma2_rn(q.xy, dx, __ffma2_rn(q.yy, dy, __fmul2_rn(q.yz, dz)));
  const float2 sz = __ffma2_rn(q.xz, dx, __ffma2_rn(q.yz, dy, __fmul2_rn(q.zz, dz)));
  const float2 dsd = __ffma2_rn(dx, sx, __ffma2_rn(dy, sy, __fmul2_rn(dz, sz)));
  // radial coefficient m inv^3 + [(15/2) dsd inv^2 - (3/2) tr] inv^5 (q.tr holds -(3/2) tr S)
  const float2 t = __ffma2_rn(dsd, __fmul2_rn(f2(7.5f), inv2), q.tr);
  float2 cw = __ffma2_rn(t, inv5, __fmul2_rn(s.m, inv3));
  float2 e = __fmul2_rn(f2(-3.f), inv5);
  cw = make_float2(on0 ? cw.x : 0.f, on1 ? cw.y : 0.f);
  e = make_float2(on0 ? e.x : 0.f, on1 ? e.y : 0.f);
  ax = __ffma2_rn(cw, dx, __ffma2_rn(e, sx, ax));
  ay = __ffma2_rn(cw, dy, __ffma2_rn(e, sy, ay));
  az = __ffma2_rn(cw, dz, __ffma2_rn(e, sz, az));
}

// Entries [0, cnt) of a pair list; an odd count is padded with a massless
// entry (it adds exactly 0).
template <bool kSoft, bool kQuad>
__device__ __forceinline__ void dense_full(V0Smem<kQuad>& S, int nf, const Target& T, Acc& a, int lane) {
  if constexpr (kQuad) {
    if (nf & 1) {
      if (lane == 0) {
        S.frec[nf >> 1].put(1, make_float4(0.f, 0.f, 0.f, 0.f));
        S.fq[nf >> 1].put(1, make_float4(0.f, 0.f, 0.f, 0.f), make_float4(0.f, 0.f, 0.f, 0.f));
      }
      __syncwarp();
    }
    const float2 nx = f2(-T.x), ny = f2(-T.y), nz = f2(-T.z), e2 = f2(T.eps2);
    float2 ax = f2(0.f), ay = f2(0.f), az = f2(0.f);
    for (int p = 0; p < (nf + 1) >> 1; ++p) {
      const RecPair s = S.frec[p];
      interact2_quad<kSoft>(ax, ay, az, s, S.fq[p], true, true, nx, ny, nz, e2);
    }
    a.x += ax.x + ax.y;
    a.y += ay.x + ay.y;
    a.z += az.x + az.y;
  } else {
    if (nf & 1) {
      if (lane == 0) S.frec[nf >> 1].put(1, make_float4(0.f, 0.f, 0.f, 0.f));
      __syncwarp();
    }
    const float2 nx = f2(-T.x), ny = f2(-T.y), nz = f2(-T.z), e2 = f2(T.eps2);
    float2 ax = f2(0.f), ay = f2(0.f), az = f2(0.f);
#pragma unroll kFUnroll
    for (int p = 0; p < (nf + 1) >> 1; ++p) {
      const RecPair s = S.frec[p];
      interact2<kSoft>(ax, ay, az, s, s.m, nx, ny, nz, e2);
    }
    a.x += ax.x + ax.y;
    a.y += ay.x + ay.y;
    a.z += az.x + az.y;
  }
  a.n += uint32_t(nf);
}

template <bool kSoft, bool kQuad>
__device__ __forceinline__ void dense_part(V0Smem<kQuad>& S, int np, const Target& T, Acc& a, int lane) {
  if constexpr (kQuad) {
    if (np & 1) {
      if (lane == 0) {
        S.prec[np >> 1].put(1, make_float4(0.f, 0.f, 0.f, 0.f));
        S.pq[np >> 1].put(1, make_float4(0.f, 0.f, 0.f, 0.f), make_float4(0.f, 0.f, 0.f, 0.f));
        S.pmsk[np] = 0u;
      }
      __syncwarp();
    }
    const float2 nx = f2(-T.x), ny = f2(-T.y), nz = f2(-T.z), e2 = f2(T.eps2);
    float2 ax = f2(0.f), ay = f2(0.f), az = f2(0.f);
    uint32_t cnt = 0;
    for (int p = 0; p < (np + 1) >> 1; ++p) {
      const RecPair s = S.prec[p];
      const uint2 mk = *reinterpret_cast<const uint2*>(&S.pmsk[2 * p]);
      const bool on0 = (mk.x >> lane) & 1u, on1 = (mk.y >> lane) & 1u;
      interact2_quad<kSoft>(ax, ay, az, s, S.pq[p], on0, on1, nx, ny, nz, e2);
      cnt += uint32_t(on0) + uint32_t(on1);
    }
    a.x += ax.x + ax.y;
    a.y += ay.x + ay.y;
    a.z += az.x + az.y;
    a.n += cnt;
  } else {
    if (np & 1) {
      if (lane == 0) {
        S.prec[np >> 1].put(1, make_float4(0.f, 0.f, 0.f, 0.f));
        S.pmsk[np] = 0u;
      }
      __syncwarp();
    }
    const float2 nx = f2(-T.x), ny = f2(-T.y), nz = f2(-T.z), e2 = f2(T.eps2);
    float2 ax = f2(0.f), ay = f2(0.f), az = f2(0.f);
    uint32_t cnt = 0;
#pragma unroll kPUnroll
    for (int p = 0; p < (np + 1) >> 1; ++p) {
      const RecPair s = S.prec[p];
      const uint2 mk = *reinterpret_cast<const uint2*>(&S.pmsk[2 * p]);
      const bool on0 = (mk.x >> lane) & 1u, on1 = (mk.y >> lane) & 1u;
      interact2<kSoft>(ax, ay, az, s, make_float2(on0 ? s.m.x : 0.f, on1 ? s.m.y : 0.f), nx, ny, nz, e2);
      cnt += uint32_t(on0) + uint32_t(on1);
    }
    a.x += ax.x + ax.y;
    a.y += ay.x + ay.y;
    a.z += az.x + az.y;
    a.n += cnt;
  }
}

// NEXT-2 FP64 mode dense phase: fp64 records, fp64 arithmetic.
#ifndef NBODY_F64_UNROLL
#define NBODY_F64_UNROLL 2
#endif
constexpr int kUnroll64 = NBODY_F64_UNROLL;

template <bool kSoft>
__device__ __forceinline__ void dense_full64(V0Smem<false, true>& S, int nf, const Target& T, AccD& a) {
#pragma unroll kUnroll64
  for (int e = 0; e < nf; ++e) {
    const double4 s = S.frec64[e];
    interact64<kSoft>(a, s, s.w, T);
  }
  a.n += uint32_t(nf);
}

template <bool kSoft>
__device__ __forceinline__ void dense_part64(V0Smem<false, true>& S, int np, const Target& T, AccD& a, int lane) {
  uint32_t cnt = 0;
#pragma unroll kUnroll64
  for (int e = 0; e < np; ++e) {
    const double4 s = S.prec64[e];
    const bool on = (S.pmsk[e] >> lane) & 1u;
    interact64<kSoft>(a, s, on ? s.w : 0.0, T);
    cnt += on;
  }
  a.n += cnt;
}

#ifndef NBODY_V0_MINB_F64
#define NBODY_V0_MINB_F64 7
#endif

template <bool kSoft, bool kQuad, bool kF64>
__global__ __launch_bounds__(32 * kV0Warps, kF64 ? NBODY_V0_MINB_F64 : NBODY_V0_MINB) void k_force_grouped(
    const ForceParams P) {
  static_assert(!(kQuad && kF64), "FP64 mode is monopole only");
  using AccT = typename std::conditional<kF64, AccD, Acc>::type;
  __shared__ V0Smem<kQuad, kF64> s_all[kV0Warps];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  V0Smem<kQuad, kF64>& S = s_all[w];
#if NBODY_SMEM_TOP > 0
  // design experiment (north star item 4, rejected: DESIGN.md "top levels in
  // shared memory"): the records and filter thresholds of the top
  // NBODY_SMEM_TOP levels (ids < 2^k) staged in shared memory for the box
  // phase, loaded once per block
  constexpr uint32_t kTop = 1u << NBODY_SMEM_TOP;
  __shared__ float4 s_trec[kTop];
  __shared__ float2 s_trc[kTop];
  for (uint32_t i = threadIdx.x; i < kTop; i += blockDim.x)
    if (i < (2u << P.t.L)) {
      s_trec[i] = __ldg(P.t.rec + i);
      s_trc[i] = __ldg(P.t.rc + i);
    }
  __syncthreads();
#endif
  const float4* qf = kQuad ? in_reg(P.t.qf) : nullptr;
#ifndef NBODY_GROUP
#define NBODY_GROUP 32
#endif
  // design experiment: NBODY_GROUP < 32 targets per warp (lanes >= NBODY_GROUP idle)
  int64_t tb, te;
  owned_range(P, tb, te);
  const int64_t k0 = tb + (int64_t(blockIdx.x) * kV0Warps + w) * NBODY_GROUP;
  const int64_t k = k0 + lane;
  const bool active = k < te && lane < NBODY_GROUP;
  const uint32_t amask = __ballot_sync(kFull, active);
  if (amask == 0) return;
  const Target T = load_target<kF64>(P, k, active);
  AccT a;
  const uint32_t lt = (1u << lane) - 1u;
  const Walk W = make_walk(P);
  const float4* tfp = in_reg(P.t.tf);
  const uint32_t leaf0 = W.leaf0;
  const uint32_t n = W.n;
  const int L = W.L;
  const uint32_t kid = leaf0 + uint32_t(k);
  const uint32_t kid0 = leaf0 + uint32_t(k0);
  // group box over the active lanes (exact fp32 min/max, used in fp64)
  const float inf = __int_as_float(0x7f800000);
  const float blx = warp_minf(active ? T.x : inf), bhx = warp_maxf(active ? T.x : -inf);
  const float bly = warp_minf(active ? T.y : inf), bhy = warp_maxf(active ? T.y : -inf);
  const float blz = warp_minf(active ? T.z : inf), bhz = warp_maxf(active ? T.z : -inf);
  // transposed-test frame: reference g = box midpoint, x' = fl(x - g), and
  // bR >= |x - g| for every target (tfilter_prep)
  const float gx = 0.5f * blx + 0.5f * bhx, gy = 0.5f * bly + 0.5f * bhy, gz = 0.5f * blz + 0.5f * bhz;
  float kk1, kk0;
  {
    // x' = fl32(x - g) (FP64 mode: of the exact fp64 difference)
    const float ux = !active ? 0.f : kF64 ? float(T.x64 - double(gx)) : T.x - gx;
    const float uy = !active ? 0.f : kF64 ? float(T.y64 - double(gy)) : T.y - gy;
    const float uz = !active ? 0.f : kF64 ? float(T.z64 - double(gz)) : T.z - gz;
    const double u2 = fma(double(uz), double(uz), fma(double(uy), double(uy), double(ux) * double(ux)));
    TgtPair& tp = S.tgt[lane >> 1];
    reinterpret_cast<float*>(&tp.px)[lane & 1] = 2.f * ux;
    reinterpret_cast<float*>(&tp.py)[lane & 1] = 2.f * uy;
    reinterpret_cast<float*>(&tp.pz)[lane & 1] = 2.f * uz;
    reinterpret_cast<float*>(&tp.q)[lane & 1] = float(-u2);
    if constexpr (kF64)
      S.tpos64[lane] = make_double4(T.x64, T.y64, T.z64, 0.0);
    else
      S.tpos[lane] = make_float4(T.x, T.y, T.z, 0.f);
    // b >= |x - g| = |x'| (1 + O(u)): 4e-7 > 2u + rounding of the bound
    const float b = __fmul_ru(warp_maxf(__fsqrt_ru(__double2float_ru(u2))), 1.f + 4e-7f);
    const float R = P.grid->R;
    kk1 = __fmaf_ru(13.f, b, __fmul_ru(5e-7f, R));
    kk0 = __fmaf_ru(__fmul_ru(7.f, b), b, __fmul_ru(__fmul_ru(2e-6f, b), R));
  }

  int na = 1, nt = 0, nf = 0, np = 0;
#ifdef NBODY_K6_STATS
  unsigned long long st[kK6Stats] = {};
  int sq[4] = {0, 0, 0, 0}, sh[2] = {0, 0}, s8[8] = {}, s16[16] = {}, s32 = 0;
  int lq[4] = {0, 0, 0, 0}, lh[2] = {0, 0}, lg = 0;  // quarter-local / half-local / general partial entries
  // boxes of the 128- and 256-target super-groups (block-level box phase study)
  float sb[2][6];
  for (int w2 = 0; w2 < 2; ++w2) {
    const int64_t span = w2 ? 256 : 128;
    const int64_t g0 = tb + ((k0 - tb) / span) * span;
    float lo[3] = {inf_stat(), inf_stat(), inf_stat()}, hi[3] = {-inf_stat(), -inf_stat(), -inf_stat()};
    for (int64_t kk = g0 + lane; kk < g0 + span && kk < te; kk += 32) {
      const float4 q = P.leaves[kk];
      lo[0] = fminf(lo[0], q.x); lo[1] = fminf(lo[1], q.y); lo[2] = fminf(lo[2], q.z);
      hi[0] = fmaxf(hi[0], q.x); hi[1] = fmaxf(hi[1], q.y); hi[2] = fmaxf(hi[2], q.z);
    }
    for (int d = 0; d < 3; ++d) { sb[w2][d] = warp_minf(lo[d]); sb[w2][3 + d] = warp_maxf(hi[d]); }
  }
  // boxes of the four 8-target quarters of this warp (T pre-test study)
  float qb[4][6];
  {
    const float tx = active ? T.x : inf_stat(), ty = active ? T.y : inf_stat(), tz = active ? T.z : inf_stat();
    const float ux = active ? T.x : -inf_stat(), uy = active ? T.y : -inf_stat(), uz = active ? T.z : -inf_stat();
    for (int q = 0; q < 4; ++q) {
      float v[6] = {tx, ty, tz, ux, uy, uz};
      for (int d = 0; d < 6; ++d) {
        float x = v[d];
        for (int o = 4; o > 0; o >>= 1) {
          const float y = __shfl_xor_sync(kFull, x, o);
          x = d < 3 ? fminf(x, y) : fmaxf(x, y);
        }
        qb[q][d] = __shfl_sync(kFull, x, 8 * q);
      }
    }
  }
#endif
  K6STAT(0, 1);
  // Super-group lists (K6a): start from the frontier of this warp's super-
  // group instead of the root, after the nodes every target of the super-
  // group accepts (every target of this warp then accepts them too, and
  // every frontier node was opened by all of them with all its ancestors,
  // so the lists are the ones the walk from the root produces).
  // (rank ranges start at multiples of kSG [A21], so super-groups are the
  // same absolute slot ranges on any partition: results bit-identical to one GPU)
  const uint32_t sgi = kSG > 0 ? uint32_t((k0 - tb) / kSG) : 0u;
  int n_acc = -1;
  {
    int2 sgc = make_int2(-1, -1);
    if (kSG > 0 && P.sg_cnt) sgc = P.sg_cnt[sgi];
    K6STAT(49, sgc.x < 0 ? 1u : 0u);  // super-group lists overflowed: this warp walks from the root
    n_acc = sgc.x;
    if (lane == 0) {
      if (sgc.x < 0) S.astk[0] = 1u;
      S.sg_next = 0;
      S.sg_nfr = sgc.x < 0 ? 0 : sgc.y;
    }
    if (sgc.x >= 0) na = 0;
  }
  __syncwarp();

  // Append (record r, lane mask msk) to the dense lists: full when every
  // active lane interacts with it.
  // active lane interacts with it.  id: the node (quadrupole source), 0 for a body.
  // g: the node id (FP64 mode reads its fp64 record rec64[g]).
  auto append = [&](bool want, const float4& r, uint32_t msk, uint32_t id, uint32_t g) {
    const bool full = want && msk == amask;
    const bool part = want && msk != amask;
    const uint32_t bf = __ballot_sync(kFull, full);
    const uint32_t bp = __ballot_sync(kFull, part);
    float4 q0 = make_float4(0.f, 0.f, 0.f, 0.f), q1 = q0;  // NEXT-4: the node's moments (0 for a body)
    if constexpr (kQuad) {
      if ((full || part) && id) {
        q0 = __ldg(qf + 2 * size_t(id));
        q1 = __ldg(qf + 2 * size_t(id) + 1);
      }
    }
    if (full) {
      const int pos = nf + __popc(bf & lt);
      if constexpr (kF64)
        S.frec64[pos] = P.t.rec64[g];
      else
        NB_CHECK(pos < S.kF);
        S.frec[pos >> 1].put(pos & 1, r);
      if constexpr (kQuad) S.fq[pos >> 1].put(pos & 1, q0, q1);
    }
    if (part) {
      const int pos = np + __popc(bp & lt);
      if constexpr (kF64)
        S.prec64[pos] = P.t.rec64[g];
      else
        S.prec[pos >> 1].put(pos & 1, r);
      NB_CHECK(pos < S.kP);
      S.pmsk[pos] = msk;
      if constexpr (kQuad) S.pq[pos >> 1].put(pos & 1, q0, q1);
    }
    nf += __popc(bf);
    np += __popc(bp);
    K6STAT(5, __popc(bf));
    K6STAT(6, __popc(bp));
    K6STAT(7, __reduce_add_sync(kFull, part ? __popc(msk) : 0u));
    K6STAT(32, __reduce_add_sync(kFull, part && __popc(msk) == 1));
    K6STAT(33, __reduce_add_sync(kFull, part && __popc(msk) == 2));
    K6STAT(34, __reduce_add_sync(kFull, part && __popc(msk) <= 4));
    K6STAT(35, __reduce_add_sync(kFull, part && __popc(msk) <= 8));
    K6STAT(8, __popc(bf) * __popc(amask));
#ifdef NBODY_K6_STATS
    {
      const uint32_t q0 = __ballot_sync(kFull, part && (msk & 0xffu)), q1 = __ballot_sync(kFull, part && (msk & 0xff00u));
      const uint32_t q2 = __ballot_sync(kFull, part && (msk & 0xff0000u)),
                     q3 = __ballot_sync(kFull, part && (msk & 0xff000000u));
      const uint32_t h0 = __ballot_sync(kFull, part && (msk & 0xffffu)), h1 = __ballot_sync(kFull, part && (msk >> 16));
      const int nq = __popc(q0) + __popc(q1) + __popc(q2) + __popc(q3);
      K6STAT(19, nq);
      K6STAT(20, __reduce_add_sync(kFull, part && (((msk & 0xffu) == msk) || ((msk & 0xff00u) == msk) ||
                                                     ((msk & 0xff0000u) == msk) || ((msk & 0xff000000u) == msk))));
      K6STAT(21, __popc(h0) + __popc(h1));
      sq[0] += __popc(q0); sq[1] += __popc(q1); sq[2] += __popc(q2); sq[3] += __popc(q3);
      sh[0] += __popc(h0); sh[1] += __popc(h1);
      for (int j = 0; j < 8; ++j) s8[j] += __popc(__ballot_sync(kFull, part && ((msk >> (4 * j)) & 0xfu)));
      for (int j = 0; j < 16; ++j) s16[j] += __popc(__ballot_sync(kFull, part && ((msk >> (2 * j)) & 0x3u)));
      s32 += part ? 0 : 0;
      {
        const bool ql = part && (((msk & 0xffu) == msk) || ((msk & 0xff00u) == msk) || ((msk & 0xff0000u) == msk) ||
                                 ((msk & 0xff000000u) == msk));
        const bool hl = part && !ql && (((msk & 0xffffu) == msk) || ((msk >> 16) << 16) == msk);
        const int q = msk & 0xffffu ? (msk & 0xffu ? 0 : 1) : (msk & 0xff0000u ? 2 : 3);
        for (int j = 0; j < 4; ++j) lq[j] += __popc(__ballot_sync(kFull, ql && q == j));
        lh[0] += __popc(__ballot_sync(kFull, hl && (msk & 0xffffu)));
        lh[1] += __popc(__ballot_sync(kFull, hl && !(msk & 0xffffu)));
        lg += __popc(__ballot_sync(kFull, part && !ql && !hl));
      }
      for (int j = 0; j < 32; ++j) {
        const uint32_t mj = __shfl_sync(kFull, msk, j);
        const bool pj = __shfl_sync(kFull, part, j);
        s32 += pj && ((mj >> lane) & 1u);
      }
    }
#endif
  };
  auto flush = [&](bool all) {
    __syncwarp();
    if (nf > S.kF - 32 || (all && nf > 0)) {
      if constexpr (kF64)
        dense_full64<kSoft>(S, nf, T, a);
      else
        dense_full<kSoft, kQuad>(S, nf, T, a, lane);
      K6STAT(10, 1);
      K6STAT(11, (nf + 1) >> 1);
      nf = 0;
    }
    if (np > S.kP - 32 || (all && np > 0)) {
      if constexpr (kF64)
        dense_part64<kSoft>(S, np, T, a, lane);
      else
        dense_part<kSoft, kQuad>(S, np, T, a, lane);
      K6STAT(12, 1);
      K6STAT(13, (np + 1) >> 1);
#ifdef NBODY_K6_STATS
      K6STAT(37, max(max(lq[0], lq[1]), max(lq[2], lq[3])));
      K6STAT(38, max(lh[0], lh[1]));
      K6STAT(39, lg);
      lq[0] = lq[1] = lq[2] = lq[3] = lh[0] = lh[1] = lg = 0;
      K6STAT(22, max(max(sq[0], sq[1]), max(sq[2], sq[3])));
      K6STAT(23, max(sh[0], sh[1]));
      sq[0] = sq[1] = sq[2] = sq[3] = sh[0] = sh[1] = 0;
      {
        int m8 = 0, m16 = 0;
        for (int j = 0; j < 8; ++j) { m8 = max(m8, s8[j]); s8[j] = 0; }
        for (int j = 0; j < 16; ++j) { m16 = max(m16, s16[j]); s16[j] = 0; }
        K6STAT(26, m8);
        K6STAT(27, m16);
        K6STAT(28, __reduce_max_sync(kFull, uint32_t(s32)));
        s32 = 0;
      }
#endif
      np = 0;
    }
    __syncwarp();
  };

  if (n_acc > 0) {  // the super-group's accepted nodes: full dense entries
    const uint32_t* al = P.sg_acc + size_t(sgi) * kSGAcc;
    for (int i = 0; i < n_acc; i += 32) {
      const bool v = i + lane < n_acc;
      const uint32_t g = v ? __ldg(al + i + lane) : 0u;
      const float4 r = v ? __ldg(W.rec + g) : make_float4(0.f, 0.f, 0.f, 0.f);
      append(v, r, amask, g, g);
      flush(false);
    }
  }
  while (true) {
    // Refill the box stack from the super-group frontier whenever it holds
    // less than one batch (the chunk goes below the nodes still stacked, so
    // box batches stay full); each chunk is popped in list order (the super-
    // group walk's discovery order, coarser nodes first): -0.5 % and -0.2 %
    // K6 against refilling an empty stack popped from the chunk's end
    // (profiles/r02_ab_k6.md).
    if (na < 32 && S.sg_next < S.sg_nfr) {
      const int next = S.sg_next;
      const int take = min(S.sg_nfr - next, S.kA - 32 - na);  // after a 32-node pop, room for 64 pushes
      const uint32_t keep = lane < na ? S.astk[lane] : 0u;
      __syncwarp();
      NB_CHECK(take + na <= S.kA);
      if (lane < na) S.astk[take + lane] = keep;
      const uint32_t* fl = P.sg_fr + size_t(sgi) * kSGFr + next;
      for (int i = lane; i < take; i += 32) S.astk[take - 1 - i] = __ldg(fl + i);
      __syncwarp();
      if (lane == 0) S.sg_next = next + take;
      na += take;
    }
    if (nt >= 32 || (na == 0 && nt > 0)) {
      // ---- T: transposed classification of up to 32 (node, mask) entries
      const int take = nt < 32 ? nt : 32;
      const int base = nt - take;
      K6STAT(3, 1);
      K6STAT(4, take);
      K6STAT(15, take < 32);
      const bool has = lane < take;
      const uint2 e = has ? S.tstk[base + lane] : make_uint2(leaf0, 0u);
      __syncwarp();
      nt = base;
      const uint32_t g = e.x, m = e.y;
      const float4 r = __ldg(W.rec + g);
      float cx = 0.f, cy = 0.f, cz = 0.f;
      float KA = inf, KO = inf;  // leaves: always interact, never open
      if (g < leaf0) tfilter_prep(r, __ldg(tfp + g), gx, gy, gz, kk1, kk0, cx, cy, cz, KA, KO);
      uint32_t am = 0u, rm = 0u;
      {
        // S = 2 c'.x' - |x'|^2; accept iff S < KA  <=>  S - KA < 0, open iff
        // S > KO  <=>  KO - S < 0: one exact rounding each (a nonzero
        // difference keeps its sign; x - x = +0; infinite thresholds give
        // infinities of the right sign), so the sign bits are the
        // comparisons, shifted into the masks from bit 31 down.
        const float2 nKA = f2(-KA), vKO = f2(KO), m1 = f2(-1.f);
#pragma unroll
        for (int t = 15; t >= 0; --t) {  // two targets per packed operation
          const float4 pxy = *reinterpret_cast<const float4*>(&S.tgt[t].px);
          const float4 pzq = *reinterpret_cast<const float4*>(&S.tgt[t].pz);
          const float2 sv = __ffma2_rn(make_float2(pxy.x, pxy.y), f2(cx),
                                       __ffma2_rn(make_float2(pxy.z, pxy.w), f2(cy),
                                                  __ffma2_rn(make_float2(pzq.x, pzq.y), f2(cz),
                                                             make_float2(pzq.z, pzq.w))));
          const float2 sa = __fadd2_rn(sv, nKA);      // S - KA
          const float2 sr = __ffma2_rn(sv, m1, vKO);  // KO - S
          am = __funnelshift_l(__float_as_uint(sa.y), am, 1);
          am = __funnelshift_l(__float_as_uint(sa.x), am, 1);
          rm = __funnelshift_l(__float_as_uint(sr.y), rm, 1);
          rm = __funnelshift_l(__float_as_uint(sr.x), rm, 1);
        }
      }
      am &= m;
      rm &= m;
#ifdef NBODY_K6_STATS
      {
        // would the box of the quarters m touches decide this node for all of m?
        float lo[3] = {inf_stat(), inf_stat(), inf_stat()}, hi[3] = {-inf_stat(), -inf_stat(), -inf_stat()};
        for (int q = 0; q < 4; ++q)
          if ((m >> (8 * q)) & 0xffu)
            for (int d = 0; d < 3; ++d) { lo[d] = fminf(lo[d], qb[q][d]); hi[d] = fmaxf(hi[d], qb[q][3 + d]); }
        const bool inner = has && g < leaf0;
        const float2 c = inner ? __ldg(W.rc + g) : make_float2(0.f, 0.f);
        const float ax0 = lo[0] - r.x, ax1 = r.x - hi[0], ay0 = lo[1] - r.y, ay1 = r.y - hi[1];
        const float az0 = lo[2] - r.z, az1 = r.z - hi[2];
        const float mx = fmaxf(0.f, fmaxf(ax0, ax1)), my = fmaxf(0.f, fmaxf(ay0, ay1)), mz = fmaxf(0.f, fmaxf(az0, az1));
        const float Mx = fmaxf(fabsf(ax0), fabsf(ax1)), My = fmaxf(fabsf(ay0), fabsf(ay1)), Mz = fmaxf(fabsf(az0), fabsf(az1));
        const float bmin2 = fmaf(mz, mz, fmaf(my, my, mx * mx)), bmax2 = fmaf(Mz, Mz, fmaf(My, My, Mx * Mx));
        const bool dec = inner && (bmin2 * (1.f - 4e-6f) > c.y || bmax2 * (1.f + 4e-6f) < c.x);
        K6STAT(50, __reduce_add_sync(kFull, inner && m == amask ? 1u : 0u));
        K6STAT(51, __reduce_add_sync(kFull, inner && m == amask && rm == m ? 1u : 0u));
        K6STAT(46, __reduce_add_sync(kFull, dec ? 1u : 0u));
        K6STAT(47, __reduce_add_sync(kFull, inner ? 1u : 0u));
        // batches in which every internal node would be decided
        K6STAT(48, __all_sync(kFull, dec || !inner) ? 1u : 0u);
      }
#endif
      uint32_t und = m & ~(am | rm);
      K6STAT(9, __reduce_add_sync(kFull, __popc(und)));
      K6STAT(16, __reduce_add_sync(kFull, has && (((m & 0xffu) == m) || ((m & 0xff00u) == m) ||
                                                  ((m & 0xff0000u) == m) || ((m & 0xff000000u) == m))));
      K6STAT(17, __reduce_add_sync(kFull, has && (((m & 0xffffu) == m) || ((m >> 16) << 16) == m)));
      K6STAT(18, __reduce_add_sync(kFull, has ? __popc(m) : 0u));
      K6STAT(24, __reduce_add_sync(kFull, has ? __popc(am) : 0u));
      K6STAT(29, __reduce_add_sync(kFull, has && g >= leaf0));
      K6STAT(31, __reduce_add_sync(kFull, has && g < leaf0 && (am == m || (rm == m))));
      K6STAT(30, __reduce_add_sync(kFull, has && g >= leaf0 / 2 && g < leaf0));
      K6STAT(25, __reduce_add_sync(kFull, has ? __popc(rm) : 0u));
      if (__any_sync(kFull, und != 0u)) {  // rare: exact fp64 decisions
        if (und) {
          const double4 pd = W.pred[g];
          do {
            const int t = __ffs(int(und)) - 1;
            bool acc;
            if constexpr (kF64) {
              const double4 tp = S.tpos64[t];
              acc = opening_accept64(pd, tp.x, tp.y, tp.z, T.th2);
            } else {
              const float4 tp = S.tpos[t];
              acc = opening_accept64(pd, tp.x, tp.y, tp.z, T.th2);
            }
            if (acc) am |= 1u << t; else rm |= 1u << t;
            und &= und - 1u;
          } while (und);
        }
      }
      if (g >= leaf0 && g - kid0 < 32u) am &= ~(1u << (g - kid0));  // a leaf never acts on itself
      append(am != 0u, r, am, g < leaf0 ? g : 0u, g);
      // children of opened nodes, with the mask of the targets that opened them
      const int l = L - 31 + __clz(int(g));
      const bool two = rm && (((2u * g + 1u) << (l - 1)) - leaf0) < n;
#if NBODY_LEAF_DIRECT
      // Children that are leaves are accepted by every target that reaches
      // them (except a target by itself), so they go straight to the dense
      // lists with the opening mask instead of through another T slot.
      const bool lv = rm != 0u && l == 1;
      if (__any_sync(kFull, lv)) {
        float4 ra = make_float4(0.f, 0.f, 0.f, 0.f), rb = ra;
        if (lv && !kF64) load_pair(W.rec + 2u * g, ra, rb);  // ids < 2^(L+1): in bounds
        const uint32_t ca = 2u * g, cb = ca + 1u;
        uint32_t ma = lv ? rm : 0u, mb = lv && two ? rm : 0u;
        if (ca - kid0 < 32u) ma &= ~(1u << (ca - kid0));
        if (cb - kid0 < 32u) mb &= ~(1u << (cb - kid0));
        flush(false);
        append(ma != 0u, ra, ma, 0u, ca);
        flush(false);
        append(mb != 0u, rb, mb, 0u, cb);
      }
      const bool push = rm != 0u && nt + 64 <= S.kT && !lv;
      const bool room = nt + 64 <= S.kT || lv;
#else
      const bool room = nt + 64 <= S.kT;
      const bool push = rm != 0u && room;
#endif
      const uint32_t b1 = __ballot_sync(kFull, push);
      const uint32_t b2 = __ballot_sync(kFull, push && two);
      if (push) {
        const int pos = nt + __popc(b1 & lt) + __popc(b2 & lt);
        NB_CHECK(pos + int(two) < S.kT);
        S.tstk[pos] = make_uint2(2u * g, rm);
        if (two) S.tstk[pos + 1] = make_uint2(2u * g + 1u, rm);
      }
      nt += __popc(b1) + __popc(b2);
      flush(false);
      // no room (never observed at the sizes we run): walk those subtrees per lane
      uint32_t spill = __ballot_sync(kFull, rm != 0u && !room);
      while (spill) {
        const int src = __ffs(int(spill)) - 1;
        K6STAT(14, 1);
        spill &= spill - 1u;
        const uint32_t gs = __shfl_sync(kFull, g, src);
        const uint32_t ms = __shfl_sync(kFull, rm, src);
        mask_walk<kQuad>(W, T, kid, a, lane, 2u * gs, ms);
        const int ls = L - 31 + __clz(int(gs));
        if ((((2u * gs + 1u) << (ls - 1)) - leaf0) < n) mask_walk<kQuad>(W, T, kid, a, lane, 2u * gs + 1u, ms);
      }
    } else if (na > 0) {
      // ---- A: box classification of up to 32 nodes reached by every lane
      const int take = na < 32 ? na : 32;
      const int base = na - take;
      K6STAT(1, 1);
      K6STAT(2, take);
      const bool has = lane < take;
      const uint32_t g = has ? S.astk[base + lane] : 0u;
      __syncwarp();
      na = base;
      const bool guard = na + 64 > S.kA;
      int cls = 0;  // 1 dense, 2 expand, 3 transposed
#ifdef NBODY_K6_STATS
      bool guard_open = false;
      int sdec[2] = {0, 0};
#endif
      float4 r = make_float4(0.f, 0.f, 0.f, 0.f);
      bool two = false;
      if (has) {
        if (g >= leaf0) {
          cls = 1;
          r = __ldg(W.rec + g);
        } else {
          // fp32 bounds of |c32 - x|^2 over the box against the node's filter
          // thresholds.  Both the box bound and every target's filter value
          // are fp32 evaluations from the same c32, equal to the exact
          // |c32 - x|^2 within 5u each, so Dmin2 (1 - 4e-6) > hi => every
          // target's d2 > hi => all accept; Dmax2 (1 + 4e-6) < lo => all open
          // (DESIGN.md "fp32 filter").
#if NBODY_SMEM_TOP > 0
          const bool top = g < kTop;
          r = top ? s_trec[g] : __ldg(W.rec + g);
          const float2 c = top ? s_trc[g] : __ldg(W.rc + g);
#else
          r = __ldg(W.rec + g);
          const float2 c = __ldg(W.rc + g);
#endif
          const float ax0 = blx - r.x, ax1 = r.x - bhx;
          const float ay0 = bly - r.y, ay1 = r.y - bhy;
          const float az0 = blz - r.z, az1 = r.z - bhz;
          const float nx = fmaxf(0.f, fmaxf(ax0, ax1)), ny = fmaxf(0.f, fmaxf(ay0, ay1)),
                      nz = fmaxf(0.f, fmaxf(az0, az1));
          const float fx = fmaxf(fabsf(ax0), fabsf(ax1)), fy = fmaxf(fabsf(ay0), fabsf(ay1)),
                      fz = fmaxf(fabsf(az0), fabsf(az1));
          const float dmin2 = fmaf(nz, nz, fmaf(ny, ny, nx * nx));
          const float dmax2 = fmaf(fz, fz, fmaf(fy, fy, fx * fx));
          if (dmin2 * (1.f - 4e-6f) > c.y) {
            cls = 1;
          } else if (dmax2 * (1.f + 4e-6f) < c.x && !guard) {
            cls = 2;
            const int l = L - 31 + __clz(int(g));
            two = ((2u * g + 1u) << (l - 1)) - leaf0 < n;
          } else {
            cls = 3;
#ifdef NBODY_K6_STATS
            guard_open = dmax2 * (1.f + 4e-6f) < c.x;  // an all-open node handed to T by the capacity guard
#endif
          }
#ifdef NBODY_K6_STATS
          for (int w2 = 0; w2 < 2; ++w2) {  // would the 128 / 256-target super-group box decide this node?
            const float bx0 = sb[w2][0] - r.x, bx1 = r.x - sb[w2][3], by0 = sb[w2][1] - r.y, by1 = r.y - sb[w2][4];
            const float bz0 = sb[w2][2] - r.z, bz1 = r.z - sb[w2][5];
            const float mx = fmaxf(0.f, fmaxf(bx0, bx1)), my = fmaxf(0.f, fmaxf(by0, by1)), mz = fmaxf(0.f, fmaxf(bz0, bz1));
            const float Mx = fmaxf(fabsf(bx0), fabsf(bx1)), My = fmaxf(fabsf(by0), fabsf(by1)), Mz = fmaxf(fabsf(bz0), fabsf(bz1));
            const float bmin2 = fmaf(mz, mz, fmaf(my, my, mx * mx)), bmax2 = fmaf(Mz, Mz, fmaf(My, My, Mx * Mx));
            sdec[w2] = bmin2 * (1.f - 4e-6f) > c.y ? 1 : bmax2 * (1.f + 4e-6f) < c.x ? 2 : 0;
          }
#endif
        }
      }
#ifdef NBODY_K6_STATS
      K6STAT(36, __reduce_add_sync(kFull, guard_open ? 1u : 0u));
      K6STAT(40, __reduce_add_sync(kFull, sdec[0] != 0 ? 1u : 0u));
      K6STAT(41, __reduce_add_sync(kFull, sdec[1] != 0 ? 1u : 0u));
      K6STAT(42, __reduce_add_sync(kFull, sdec[0] == 1 ? 1u : 0u));
      K6STAT(43, __reduce_add_sync(kFull, has && g < leaf0 ? 1u : 0u));
      K6STAT(44, __reduce_add_sync(kFull, cls == 1 && g < leaf0 ? 1u : 0u));
      K6STAT(45, __reduce_add_sync(kFull, cls == 2 ? 1u : 0u));
#endif
      uint32_t msk = amask;
      if (cls == 1 && g >= leaf0 && g - kid0 < 32u) msk &= ~(1u << (g - kid0));  // not on itself
      append(cls == 1, r, msk, g < leaf0 ? g : 0u, g);
      const uint32_t bt = __ballot_sync(kFull, cls == 3);
      if (cls == 3) NB_CHECK(nt + __popc(bt & lt) < S.kT);
      if (cls == 3) S.tstk[nt + __popc(bt & lt)] = make_uint2(g, amask);
      nt += __popc(bt);
      const uint32_t b1 = __ballot_sync(kFull, cls == 2);
      const uint32_t b2 = __ballot_sync(kFull, cls == 2 && two);
      if (cls == 2) {
        const int pos = na + __popc(b1 & lt) + __popc(b2 & lt);
        NB_CHECK(pos + int(two) < S.kA);
        S.astk[pos] = 2u * g;
        if (two) S.astk[pos + 1] = 2u * g + 1u;
      }
      na += __popc(b1) + __popc(b2);
      flush(false);
    } else {
      break;
    }
  }
  flush(true);
  store_result(P, tb, k, k0, active, a, lane);
#ifdef NBODY_K6_STATS
  if (lane == 0)
    for (int i = 0; i < kK6Stats; ++i) atomicAdd(&g_k6_stats[i], st[i]);
#endif
}

// ------------------------------------------------ super-group pre-pass ----
// K6a: one warp per super-group of kSG consecutive owned targets classifies
// nodes from the root against the super-group's bounding box with the box
// phase's bounds (every target accepts / every target opens / neither):
// accepted nodes go to acc, nodes it cannot decide (and leaves, whose
// self-exclusion the force warps apply) to the frontier fr, nodes every
// target opens are expanded.  Any warp of the super-group would decide
// those nodes the same way with its own (smaller) box, so the force warps
// take acc as full dense entries and continue from fr: the box-phase work
// near the root is done once per kSG targets instead of once per 32.
constexpr int kSGWarps = 4;

template <bool kF64>
__global__ __launch_bounds__(32 * kSGWarps) void k_force_sgroups(const ForceParams P) {
  __shared__ uint32_t s_stk[kSGWarps][kCapA];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int64_t tb, te;
  owned_range(P, tb, te);
  // list j of this rank: slots [tb + j kSG, tb + (j + 1) kSG) -- rank ranges
  // start at multiples of kSG [A21], so these are the same absolute super-
  // groups (hence the same lists) on any partition
  const int64_t sgi = int64_t(blockIdx.x) * kSGWarps + w;
  const int64_t g0 = tb + sgi * kSG;
  if (g0 >= te) return;
  const int64_t g1 = g0 + kSG < te ? g0 + kSG : te;
  const float inf = __int_as_float(0x7f800000);
  float lx = inf, ly = inf, lz = inf, hx = -inf, hy = -inf, hz = -inf;
  for (int64_t k = g0 + lane; k < g1; k += 32) {
    float x, y, z;
    if constexpr (kF64) {  // the force kernel's fp32 rounding of the fp64 targets
      const double4 q = P.leaves64[k];
      x = float(q.x), y = float(q.y), z = float(q.z);
    } else {
      const float4 q = P.leaves[k];
      x = q.x, y = q.y, z = q.z;
    }
    lx = fminf(lx, x), ly = fminf(ly, y), lz = fminf(lz, z);
    hx = fmaxf(hx, x), hy = fmaxf(hy, y), hz = fmaxf(hz, z);
  }
  const float blx = warp_minf(lx), bly = warp_minf(ly), blz = warp_minf(lz);
  const float bhx = warp_maxf(hx), bhy = warp_maxf(hy), bhz = warp_maxf(hz);
  const float4* rec = in_reg(P.t.rec);
  const float2* rc = in_reg(P.t.rc);
  const uint32_t leaf0 = 1u << P.t.L, n = uint32_t(P.t.n);
  const int L = P.t.L;
  uint32_t* stk = s_stk[w];
  uint32_t* acc = P.sg_acc + sgi * kSGAcc;
  uint32_t* fr = P.sg_fr + sgi * kSGFr;
  const uint32_t lt = (1u << lane) - 1u;
  int na = 1, nacc = 0, nfr = 0;
  if (lane == 0) stk[0] = 1u;
  __syncwarp();
  while (na > 0) {
    // Bounded lists (wide opening angles reach thousands of nodes per super-
    // group): once the frontier could no longer take one more batch plus the
    // whole stack, the stack itself becomes frontier and the walk stops; once
    // the accepted list is full, accepted nodes go to the frontier too.  Every
    // such node has only ancestors opened by all kSG targets, so the force
    // warps continue from it exactly as from the root (their smaller boxes
    // accept what this box accepts).  One batch adds <= 32 frontier entries
    // and <= 64 - take stack entries, hence the margin of 96.
    if (nfr + na + 96 > kSGFr) {
      NB_CHECK(nfr + na <= kSGFr);
      for (int i = lane; i < na; i += 32) fr[nfr + i] = stk[i];
      nfr += na;
      break;
    }
    const bool acc_full = nacc + 32 > kSGAcc;
    const int take = na < 32 ? na : 32;
    const int base = na - take;
    const bool has = lane < take;
    const uint32_t g = has ? stk[base + lane] : 0u;
    __syncwarp();
    na = base;
    const bool guard = na + 64 > kCapA;
    int cls = 0;  // 1 accepted by every target, 2 opened by every target, 3 frontier
    bool two = false;
    if (has) {
      if (g >= leaf0) {
        cls = 3;
      } else {
        // the force kernel's box-phase bounds
        const float4 r = __ldg(rec + g);
        const float2 c = __ldg(rc + g);
        const float ax0 = blx - r.x, ax1 = r.x - bhx;
        const float ay0 = bly - r.y, ay1 = r.y - bhy;
        const float az0 = blz - r.z, az1 = r.z - bhz;
        const float nx = fmaxf(0.f, fmaxf(ax0, ax1)), ny = fmaxf(0.f, fmaxf(ay0, ay1)),
                    nz = fmaxf(0.f, fmaxf(az0, az1));
        const float fx = fmaxf(fabsf(ax0), fabsf(ax1)), fy = fmaxf(fabsf(ay0), fabsf(ay1)),
                    fz = fmaxf(fabsf(az0), fabsf(az1));
        const float dmin2 = fmaf(nz, nz, fmaf(ny, ny, nx * nx));
        const float dmax2 = fmaf(fz, fz, fmaf(fy, fy, fx * fx));
        if (dmin2 * (1.f - 4e-6f) > c.y) {
          cls = acc_full ? 3 : 1;
        } else if (dmax2 * (1.f + 4e-6f) < c.x && !guard) {
          cls = 2;
          const int l = L - 31 + __clz(int(g));
          two = ((2u * g + 1u) << (l - 1)) - leaf0 < n;
        } else {
          cls = 3;
        }
      }
    }
    const uint32_t ba = __ballot_sync(kFull, cls == 1), bf = __ballot_sync(kFull, cls == 3);
    if (cls == 1) NB_CHECK(nacc + __popc(ba & lt) < kSGAcc);
    if (cls == 3) NB_CHECK(nfr + __popc(bf & lt) < kSGFr);
    if (cls == 1) acc[nacc + __popc(ba & lt)] = g;
    if (cls == 3) fr[nfr + __popc(bf & lt)] = g;
    nacc += __popc(ba);
    nfr += __popc(bf);
    const uint32_t b1 = __ballot_sync(kFull, cls == 2), b2 = __ballot_sync(kFull, cls == 2 && two);
    if (cls == 2) {
      const int pos = na + __popc(b1 & lt) + __popc(b2 & lt);
      NB_CHECK(pos + int(two) < kCapA);
      stk[pos] = 2u * g;
      if (two) stk[pos + 1] = 2u * g + 1u;
    }
    na += __popc(b1) + __popc(b2);
    __syncwarp();
  }
  if (lane == 0) P.sg_cnt[sgi] = make_int2(nacc, nfr);
}

}  // namespace

void launch_force_sgroups(const ForceParams& p, cudaStream_t s) {
  if (kSG <= 0 || !p.sg_cnt) return;
  const int64_t nt = p.part ? p.cap : p.t_end - p.t_begin;
  if (nt <= 0) return;
  const int64_t groups = (nt + kSG - 1) / kSG;
  const unsigned grid = unsigned((groups + kSGWarps - 1) / kSGWarps);
  if (p.t.rec64)
    k_force_sgroups<true><<<grid, 32 * kSGWarps, 0, s>>>(p);
  else
    k_force_sgroups<false><<<grid, 32 * kSGWarps, 0, s>>>(p);
}

void launch_force(const ForceParams& p, int variant, cudaStream_t s) {
  const int64_t nt = p.part ? p.cap : p.t_end - p.t_begin;
  if (nt <= 0) return;
  const int64_t warps = (nt + 31) / 32;
  const bool quad = p.t.quad;
  if (variant == 2) {  // the paper's per-body skip-list walk (monopole)
    k_force_skiplist<<<unsigned((nt + kV2Threads - 1) / kV2Threads), kV2Threads, 0, s>>>(p);
  } else if (variant == 1) {
    const unsigned grid = unsigned((warps + kV1Warps - 1) / kV1Warps);
    if (quad)
      k_force_maskstack<true><<<grid, 32 * kV1Warps, 0, s>>>(p);
    else
      k_force_maskstack<false><<<grid, 32 * kV1Warps, 0, s>>>(p);
  } else {
    const unsigned grid = unsigned(((nt + NBODY_GROUP - 1) / NBODY_GROUP + kV0Warps - 1) / kV0Warps);
    const bool soft = p.t.rec64 ? p.eps2_64 > 0.0 : p.eps2 > 0.f;
    if (p.t.rec64) {  // NEXT-2 FP64 mode (monopole, variant 0)
      if (soft)
        k_force_grouped<true, false, true><<<grid, 32 * kV0Warps, 0, s>>>(p);
      else
        k_force_grouped<false, false, true><<<grid, 32 * kV0Warps, 0, s>>>(p);
    } else if (soft && !quad)
      k_force_grouped<true, false, false><<<grid, 32 * kV0Warps, 0, s>>>(p);
    else if (!soft && !quad)
      k_force_grouped<false, false, false><<<grid, 32 * kV0Warps, 0, s>>>(p);
    else if (soft)
      k_force_grouped<true, true, false><<<grid, 32 * kV0Warps, 0, s>>>(p);
    else
      k_force_grouped<false, true, false><<<grid, 32 * kV0Warps, 0, s>>>(p);
  }
}


// Load every kernel of this file now (see preload_all in capi.cu).
void preload_force() {
  touch(k_force_grouped<false, false, false>);
  touch(k_force_grouped<false, false, true>);
  touch(k_force_grouped<false, true, false>);
  touch(k_force_grouped<true, false, false>);
  touch(k_force_grouped<true, false, true>);
  touch(k_force_grouped<true, true, false>);
  touch(k_force_maskstack<false>);
  touch(k_force_maskstack<true>);
  touch(k_force_skiplist);
  touch(k_force_sgroups<false>);
  touch(k_force_sgroups<true>);
}

}  // namespace nb
