// K6 CALCULATEFORCE over the Hilbert-sorted BVH (
// Eq. 1 P:72 with Plummer softening [A1], G = 1 [A2]).
//
// Semantics (identical to the oracle's per-body DFS): for target k, node n
// is in k's interaction list iff every proper ancestor of n fails the
// opening test for k and n passes it (or n is a leaf other than k).  The
// opening test is the fixed fp64 expression [A3][A16][A20]
//     s^2 < theta^2 * fma(dz, dz, fma(dy, dy, dx*dx)),  d = com64 - x_k,
// evaluated with explicitly rounded intrinsics, so every decision -- hence
// every interaction list -- is bit-identical to the oracle's.  The
// interaction itself is fp32 (rsqrtf + FMA) on the monopole
// ((float)com, (float)M); its summation order is free (tolerance-checked).
//
// Variant 1, warp mask-stack walk: the 32 lanes of a warp own 32
// Hilbert-consecutive targets and walk the tree together.  A shared-memory
// stack holds sibling pairs (level, pair index, lane mask of the lanes that
// reached the pair).  Each popped pair is loaded once for the whole warp
// (broadcast), every lane in the mask tests both siblings, lanes that accept
// interact immediately, and the ballots of rejecting lanes become the masks
// of the children pairs.  No lane ever visits a node it would not visit in
// its own DFS, so lists are exact; idle lanes cost issue slots only.
#include "internal.cuh"

namespace nb {
namespace {

constexpr unsigned kFull = 0xffffffffu;

__device__ __forceinline__ bool opening_accept(const double4& p, double x, double y, double z, double th2) {
  const double dx = __dsub_rn(p.x, x);
  const double dy = __dsub_rn(p.y, y);
  const double dz = __dsub_rn(p.z, z);
  const double d2 = __fma_rn(dz, dz, __fma_rn(dy, dy, __dmul_rn(dx, dx)));
  return p.w < __dmul_rn(th2, d2);
}

struct Acc {
  float x = 0.f, y = 0.f, z = 0.f;
  uint32_t n = 0;
  __device__ __forceinline__ void add(const float4& s, const float4& me, float eps2) {
    const float dx = s.x - me.x, dy = s.y - me.y, dz = s.z - me.z;
    const float r2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
    const float inv = r2 > 0.f ? rsqrtf(r2) : 0.f;  // r2 == 0 only when eps == 0: no contribution
    const float w = s.w * inv * inv * inv;
    x = fmaf(w, dx, x);
    y = fmaf(w, dy, y);
    z = fmaf(w, dz, z);
    ++n;
  }
};

constexpr int kWarpsPerBlock = 8;
constexpr int kStack = 64;

__global__ __launch_bounds__(32 * kWarpsPerBlock) void k_force_maskstack(const ForceParams P) {
  __shared__ uint32_t s_idx[kWarpsPerBlock][kStack];
  __shared__ uint32_t s_msk[kWarpsPerBlock][kStack];
  __shared__ int s_lvl[kWarpsPerBlock][kStack];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t k = P.t_begin + (int64_t(blockIdx.x) * kWarpsPerBlock + w) * 32 + lane;
  const bool active = k < P.t_end;
  const uint32_t amask = __ballot_sync(kFull, active);
  if (amask == 0) return;
  const float4 me = active ? P.leaves[k] : make_float4(0.f, 0.f, 0.f, 0.f);
  const double x64 = me.x, y64 = me.y, z64 = me.z;
  Acc a;
  const int L = P.t.L;

  int sp = 1;
  if (lane == 0) {
    s_lvl[w][0] = L;
    s_idx[w][0] = 0;
    s_msk[w][0] = amask;
  }
  __syncwarp();
  while (sp > 0) {
    --sp;
    const int l = s_lvl[w][sp];
    const uint32_t p = s_idx[w][sp];
    const uint32_t m = s_msk[w][sp];
    __syncwarp();
    const bool in = (m >> lane) & 1u;
    const int64_t jA = 2 * int64_t(p), jB = jA + 1;
    const bool hasB = jB < P.t.count[l];
    if (l == 0) {  // two leaves: exact interactions, the target excluded
      const float4 A = P.leaves[jA];
      if (in && jA != k) a.add(A, me, P.eps2);
      if (hasB) {
        const float4 B = P.leaves[jB];
        if (in && jB != k) a.add(B, me, P.eps2);
      }
      continue;
    }
    const int64_t node = P.t.off[l] + jA;
    const double4 pa = P.t.pred[node];
    const bool accA = opening_accept(pa, x64, y64, z64, P.th2);
    bool accB = false;
    if (hasB) accB = opening_accept(P.t.pred[node + 1], x64, y64, z64, P.th2);
    const uint32_t rejA = __ballot_sync(kFull, in && !accA);
    const uint32_t rejB = __ballot_sync(kFull, in && hasB && !accB);
    const bool doA = in && accA, doB = in && hasB && accB;
    if (__any_sync(kFull, doA)) {
      const float4 r = P.t.rec[node];
      if (doA) a.add(r, me, P.eps2);
    }
    if (__any_sync(kFull, doB)) {
      const float4 r = P.t.rec[node + 1];
      if (doB) a.add(r, me, P.eps2);
    }
    // children of (l, jB) then of (l, jA): the A subtree is walked first
    if (lane == 0) {
      int q = sp;
      if (rejB) { s_lvl[w][q] = l - 1; s_idx[w][q] = uint32_t(jB); s_msk[w][q] = rejB; ++q; }
      if (rejA) { s_lvl[w][q] = l - 1; s_idx[w][q] = uint32_t(jA); s_msk[w][q] = rejA; }
    }
    sp += (rejB != 0) + (rejA != 0);
    __syncwarp();
  }
  if (active) {
    P.acc[k - P.t_begin] = make_float4(a.x, a.y, a.z, 0.f);
    P.count[k - P.t_begin] = a.n;
  }
  const uint32_t tot = __reduce_add_sync(kFull, a.n);
  if (lane == 0) atomicAdd(P.total, (unsigned long long)tot);
}

}  // namespace

void launch_force(const ForceParams& p, int variant, cudaStream_t s) {
  (void)variant;
  const int64_t nt = p.t_end - p.t_begin;
  if (nt <= 0) return;
  const int64_t warps = (nt + 31) / 32;
  const unsigned grid = unsigned((warps + kWarpsPerBlock - 1) / kWarpsPerBlock);
  k_force_maskstack<<<grid, 32 * kWarpsPerBlock, 0, s>>>(p);
}

}  // namespace nb
