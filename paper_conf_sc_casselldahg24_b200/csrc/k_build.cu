// K4 permutation gather ("applying it as a permutation afterwards";
// [A11] the whole body state moves) and K5 BUILDTREEACCUMULATEMASS (P:218,
// P:221, Fig. 4; multipoles P:105).
//
// K5 reduces the two children of every node (left then right) level by
// level -- the paper's algorithm.  Moments (M, M x) are fp64 sums in that
// fixed order and the boxes exact fp32 min/max, so every node record is
// bit-identical to the oracle's [A12][A13][A16].  Per node it emits the
// opening-test record (com64, s^2), the fp32 filter thresholds and the fp32
// monopole ((float)com64, (float)M) used by K6; with NEXT-4 also the second
// moment about the COM (parallel-axis theorem, fp64, the oracle's operation
// order) [A24].
//
// Default variant: a block reduces a 1024-leaf subtree (levels 1..10) in
// shared memory and one block builds the top levels; variant 1 launches one
// kernel per level (monopole only).  Both give identical records.
#include <type_traits>

#include "internal.cuh"

namespace nb {
namespace {

__global__ __launch_bounds__(256) void k_permute(const float4* __restrict__ pm_in, const float4* __restrict__ vi_in,
                                                 const uint32_t* __restrict__ perm, int64_t n,
                                                 float4* __restrict__ pm_out, float4* __restrict__ vi_out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t p = perm[i];
  pm_out[i] = __ldg(pm_in + p);
  vi_out[i] = __ldg(vi_in + p);
}

// [A24] S_p += S_c + (M_c d_i) d_j, d = com_c - com_p, in the oracle's order.
__device__ __forceinline__ void add_second_moment(double* Sp, const double* Sc, double Mc, const double* cc,
                                                  const double* cp) {
  const double d0 = __dsub_rn(cc[0], cp[0]), d1 = __dsub_rn(cc[1], cp[1]), d2 = __dsub_rn(cc[2], cp[2]);
  const double di[6] = {d0, d1, d2, d0, d0, d1}, dj[6] = {d0, d1, d2, d1, d2, d2};
#pragma unroll
  for (int q = 0; q < 6; ++q) Sp[q] = __dadd_rn(Sp[q], __dadd_rn(Sc[q], __dmul_rn(__dmul_rn(Mc, di[q]), dj[q])));
}

// Box helpers for fp32 (float4) and fp64 (double4, NEXT-2) bounds: exact
// min/max either way.
__device__ __forceinline__ float4 box_min(float4 a, float4 b) {
  return make_float4(fminf(a.x, b.x), fminf(a.y, b.y), fminf(a.z, b.z), 0.f);
}
__device__ __forceinline__ float4 box_max(float4 a, float4 b) {
  return make_float4(fmaxf(a.x, b.x), fmaxf(a.y, b.y), fmaxf(a.z, b.z), 0.f);
}
__device__ __forceinline__ double4 box_min(double4 a, double4 b) {
  return make_double4(fmin(a.x, b.x), fmin(a.y, b.y), fmin(a.z, b.z), 0.0);
}
__device__ __forceinline__ double4 box_max(double4 a, double4 b) {
  return make_double4(fmax(a.x, b.x), fmax(a.y, b.y), fmax(a.z, b.z), 0.0);
}
__device__ __forceinline__ void store_box(const TreeView& t, int64_t node, float4 lo, float4 hi) {
  t.blo[node] = lo;
  t.bhi[node] = hi;
}
__device__ __forceinline__ void store_box(const TreeView& t, int64_t node, double4 lo, double4 hi) {
  t.blo64[node] = lo;
  t.bhi64[node] = hi;
}
__device__ __forceinline__ float4 load_lo(const TreeView& t, int64_t node, float4*) { return t.blo[node]; }
__device__ __forceinline__ float4 load_hi(const TreeView& t, int64_t node, float4*) { return t.bhi[node]; }
__device__ __forceinline__ double4 load_lo(const TreeView& t, int64_t node, double4*) { return t.blo64[node]; }
__device__ __forceinline__ double4 load_hi(const TreeView& t, int64_t node, double4*) { return t.bhi64[node]; }

// Emit node `node` with centre of mass c: the traversal records (pred, rec,
// rc, tf[, qf][, rec64]) always; the build moments, box [and S64] only when
// `keep` (needed by a parent built in another block, or by the debug views).
template <class B4>
__device__ __forceinline__ void finish_node(const TreeView& t, int64_t node, double M, double mx, double my, double mz,
                                            const double* c, B4 lo, B4 hi, bool keep,
                                            const double* S = nullptr) {
  constexpr bool kF64 = sizeof(B4) == 32;
  if (keep) {
    t.mom[node] = make_double4(M, mx, my, mz);
    store_box(t, node, lo, hi);
  }
  if (kF64) t.rec64[node] = make_double4(c[0], c[1], c[2], M);
  // [A3] s = longest side of the AABB (fp64 differences: exact for fp32
  // bounds, rounded for fp64 bounds -- the oracle's expression either way)
  double s = __dsub_rn(double(hi.x), double(lo.x));
  s = fmax(s, __dsub_rn(double(hi.y), double(lo.y)));
  s = fmax(s, __dsub_rn(double(hi.z), double(lo.z)));
  const double s2 = __dmul_rn(s, s);
  t.pred[node] = make_double4(c[0], c[1], c[2], s2);
  // Filter thresholds on the fp32 squared distance (DESIGN.md "fp32
  // filter"): |d2_fp32 - d^2| <= 1.01e-4 d^2 + A with A = 1e-9 R^2, so
  // d2 > (1 + 2e-4) s^2/theta^2 + A surely accepts and
  // d2 < (1 - 2e-4) s^2/theta^2 - A surely opens.
  float2 rc;
  const double q = t.th2 > 0.0 ? __ddiv_rn(s2, t.th2) : 0.0;  // s^2 / theta^2, once per node
  if (t.th2 > 0.0) {
    const double A = double(t.grid->abs_d2);
    rc.x = __double2float_rd((1.0 - 2e-4) * q - A);
    rc.y = __double2float_ru((1.0 + 2e-4) * q + A);
  } else {  // theta = 0 opens every node
    rc.x = rc.y = __int_as_float(0x7f800000);
  }
  t.rc[node] = rc;
  const float c0 = __double2float_rn(c[0]), c1 = __double2float_rn(c[1]), c2 = __double2float_rn(c[2]);
  t.rec[node] = make_float4(c0, c1, c2, __double2float_rn(M));
  // T-phase filter data: the fp32 residuals of the COM (com64 - c32 is exact
  // in fp64) and q = s^2 / theta^2 (+inf at theta = 0)
  t.tf[node] = make_float4(__double2float_rn(__dsub_rn(c[0], double(c0))),
                           __double2float_rn(__dsub_rn(c[1], double(c1))),
                           __double2float_rn(__dsub_rn(c[2], double(c2))),
                           t.th2 > 0.0 ? __double2float_rn(q) : __int_as_float(0x7f800000));
  if (S) {
    if (keep) {
#pragma unroll
      for (int q = 0; q < 6; ++q) t.S64[node].s[q] = S[q];
    }
    const float sxx = __double2float_rn(S[0]), syy = __double2float_rn(S[1]), szz = __double2float_rn(S[2]);
    t.qf[2 * node] = make_float4(sxx, syy, szz, __double2float_rn(S[0] + S[1] + S[2]));
    t.qf[2 * node + 1] = make_float4(__double2float_rn(S[3]), __double2float_rn(S[4]), __double2float_rn(S[5]), 0.f);
  }
}

// centre of mass = first moment / mass [A12]
__device__ __forceinline__ void node_com(double M, double mx, double my, double mz, double* c) {
  c[0] = __ddiv_rn(mx, M);
  c[1] = __ddiv_rn(my, M);
  c[2] = __ddiv_rn(mz, M);
}

// Level 1 straight from the sorted bodies: leaf moments are M = m and
// M x = m * x (exact in fp64), leaf boxes are points [A13].
__global__ __launch_bounds__(256) void k_build_level1(TreeView t, const float4* __restrict__ leaves) {
  const int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (j >= t.count[1]) return;
  const int64_t a = 2 * j, b = a + 1;
  const float4 A = __ldg(leaves + a);
  double M = double(A.w);
  double mx = __dmul_rn(double(A.w), double(A.x));
  double my = __dmul_rn(double(A.w), double(A.y));
  double mz = __dmul_rn(double(A.w), double(A.z));
  float4 lo = make_float4(A.x, A.y, A.z, 0.f), hi = lo;
  if (b < t.n) {
    const float4 B = __ldg(leaves + b);
    M = __dadd_rn(M, double(B.w));
    mx = __dadd_rn(mx, __dmul_rn(double(B.w), double(B.x)));
    my = __dadd_rn(my, __dmul_rn(double(B.w), double(B.y)));
    mz = __dadd_rn(mz, __dmul_rn(double(B.w), double(B.z)));
    lo.x = fminf(lo.x, B.x); lo.y = fminf(lo.y, B.y); lo.z = fminf(lo.z, B.z);
    hi.x = fmaxf(hi.x, B.x); hi.y = fmaxf(hi.y, B.y); hi.z = fmaxf(hi.z, B.z);
  }
  double c[3];
  node_com(M, mx, my, mz, c);
  finish_node(t, t.off[1] + j, M, mx, my, mz, c, lo, hi, true);
}

// Level l >= 2 from level l - 1.
__global__ __launch_bounds__(256) void k_build_level(TreeView t, int l) {
  const int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (j >= t.count[l]) return;
  const int64_t ca = t.off[l - 1] + 2 * j;
  const bool two = 2 * j + 1 < t.count[l - 1];
  double4 m = t.mom[ca];
  float4 lo = t.blo[ca], hi = t.bhi[ca];
  if (two) {
    const double4 mb = t.mom[ca + 1];
    const float4 lb = t.blo[ca + 1], hb = t.bhi[ca + 1];
    m.x = __dadd_rn(m.x, mb.x);
    m.y = __dadd_rn(m.y, mb.y);
    m.z = __dadd_rn(m.z, mb.z);
    m.w = __dadd_rn(m.w, mb.w);
    lo.x = fminf(lo.x, lb.x); lo.y = fminf(lo.y, lb.y); lo.z = fminf(lo.z, lb.z);
    hi.x = fmaxf(hi.x, hb.x); hi.y = fmaxf(hi.y, hb.y); hi.z = fmaxf(hi.z, hb.z);
  }
  double c[3];
  node_com(m.x, m.y, m.z, m.w, c);
  finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, c, lo, hi, true);
}

// Fused build of levels 1..top (top <= 10) over a 1024-leaf subtree per
// block: each level is reduced from the previous one in shared memory (same
// left+right fp64 order, so the records are identical to the level-by-level
// kernels); only the subtree roots (level top) keep moments/boxes in global
// memory unless keep_all (debug views).
constexpr int kFuseLevels = 10;
#ifndef NBODY_UPPER_WIDE
#define NBODY_UPPER_WIDE 3  // upper levels built by one grid each before the one-block kernel
#endif
constexpr int kFuseHalf = 1 << (kFuseLevels - 1);  // level-1 nodes per block
constexpr int kFuseThreads = 256;

template <bool kQuad>
constexpr int fuse_half() {  // level-1 nodes per block (quad: 512-leaf subtrees, 9 levels)
  return kQuad ? kFuseHalf / 2 : kFuseHalf;
}

#ifndef NBODY_BUILD_MINB
#define NBODY_BUILD_MINB 4  // 64 registers: 4 blocks per SM (0.449 -> 0.408 ms for permute + build at 1e7)
#endif
template <bool kQuad, bool kF64>
__global__ __launch_bounds__(kFuseThreads, kQuad ? 1 : NBODY_BUILD_MINB) void k_build_fused(TreeView t, const float4* __restrict__ leaves, int top,
                                                              bool keep_all) {
  using B4 = typename std::conditional<kF64, double4, float4>::type;  // box / leaf type
  constexpr int kHalf = (kQuad || kF64) ? kFuseHalf / 2 : kFuseHalf;
  __shared__ double4 s_m[kHalf];
  __shared__ B4 s_lo[kHalf];
  __shared__ B4 s_hi[kHalf];
  __shared__ double s_c[kQuad ? 3 * kHalf : 1];
  __shared__ double s_S[kQuad ? 6 * kHalf : 1];
  const B4* lv = kF64 ? reinterpret_cast<const B4*>(t.rec64 + (int64_t(1) << t.L))
                      : reinterpret_cast<const B4*>(leaves);
  const int64_t b = blockIdx.x;
  for (int q = threadIdx.x; q < kHalf; q += kFuseThreads) {
    const int64_t j = b * kHalf + q;
    if (j >= t.count[1]) continue;
    const int64_t a = 2 * j;
    const B4 A = lv[a];
    const bool two = a + 1 < t.n;
    const B4 B = two ? lv[a + 1] : A;
    double M = double(A.w);
    double mx = __dmul_rn(double(A.w), double(A.x));
    double my = __dmul_rn(double(A.w), double(A.y));
    double mz = __dmul_rn(double(A.w), double(A.z));
    B4 lo = A, hi = A;
    lo.w = 0;
    hi.w = 0;
    if (two) {
      M = __dadd_rn(M, double(B.w));
      mx = __dadd_rn(mx, __dmul_rn(double(B.w), double(B.x)));
      my = __dadd_rn(my, __dmul_rn(double(B.w), double(B.y)));
      mz = __dadd_rn(mz, __dmul_rn(double(B.w), double(B.z)));
      lo = box_min(lo, B);
      hi = box_max(hi, B);
    }
    double c[3];
    node_com(M, mx, my, mz, c);
    const bool keep = keep_all || top == 1;
    if (kQuad) {
      // leaves: com = position, S = 0 [A24]
      const double zero[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
      double S[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
      const double ca[3] = {double(A.x), double(A.y), double(A.z)};
      add_second_moment(S, zero, double(A.w), ca, c);
      if (two) {
        const double cb[3] = {double(B.x), double(B.y), double(B.z)};
        add_second_moment(S, zero, double(B.w), cb, c);
      }
      finish_node(t, t.off[1] + j, M, mx, my, mz, c, lo, hi, keep, S);
      for (int k = 0; k < 3; ++k) s_c[3 * q + k] = c[k];
      for (int k = 0; k < 6; ++k) s_S[6 * q + k] = S[k];
    } else {
      finish_node(t, t.off[1] + j, M, mx, my, mz, c, lo, hi, keep);
    }
    s_m[q] = make_double4(M, mx, my, mz);
    s_lo[q] = lo;
    s_hi[q] = hi;
  }
  __syncthreads();
  for (int l = 2; l <= top; ++l) {
    const int cnt = kHalf >> (l - 1);  // nodes of level l in this block (<= 256)
    const int q = threadIdx.x;
    const int64_t j = b * cnt + q;
    bool have = false;
    double4 m;
    B4 lo, hi;
    double c[3], S[6];
    if (q < cnt && j < t.count[l]) {
      have = true;
      const bool two = 2 * j + 1 < t.count[l - 1];
      m = s_m[2 * q];
      lo = s_lo[2 * q];
      hi = s_hi[2 * q];
      if (two) {
        const double4 mb = s_m[2 * q + 1];
        m.x = __dadd_rn(m.x, mb.x);
        m.y = __dadd_rn(m.y, mb.y);
        m.z = __dadd_rn(m.z, mb.z);
        m.w = __dadd_rn(m.w, mb.w);
        lo = box_min(lo, s_lo[2 * q + 1]);
        hi = box_max(hi, s_hi[2 * q + 1]);
      }
      node_com(m.x, m.y, m.z, m.w, c);
      if (kQuad) {
        for (int k = 0; k < 6; ++k) S[k] = 0.0;
        add_second_moment(S, &s_S[6 * (2 * q)], s_m[2 * q].x, &s_c[3 * (2 * q)], c);
        if (two) add_second_moment(S, &s_S[6 * (2 * q + 1)], s_m[2 * q + 1].x, &s_c[3 * (2 * q + 1)], c);
      }
    }
    __syncthreads();
    if (have) {
      s_m[q] = m;
      s_lo[q] = lo;
      s_hi[q] = hi;
      const bool keep = keep_all || l == top;
      if (kQuad) {
        for (int k = 0; k < 3; ++k) s_c[3 * q + k] = c[k];
        for (int k = 0; k < 6; ++k) s_S[6 * q + k] = S[k];
        finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, c, lo, hi, keep, S);
      } else {
        finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, c, lo, hi, keep);
      }
    }
    __syncthreads();
  }
}

// Levels from..L in one block (the top of the tree is small: ceil(N / 2^l)
// nodes per level); __syncthreads orders the levels.
template <bool kF64>
__global__ __launch_bounds__(1024) void k_build_upper(TreeView t, int from) {
  using B4 = typename std::conditional<kF64, double4, float4>::type;
  B4* tag = nullptr;
  for (int l = from; l <= t.L; ++l) {
    for (int64_t j = threadIdx.x; j < t.count[l]; j += blockDim.x) {
      const int64_t ca = t.off[l - 1] + 2 * j;
      const bool two = 2 * j + 1 < t.count[l - 1];
      double4 m = t.mom[ca];
      B4 lo = load_lo(t, ca, tag), hi = load_hi(t, ca, tag);
      if (two) {
        const double4 mb = t.mom[ca + 1];
        m.x = __dadd_rn(m.x, mb.x);
        m.y = __dadd_rn(m.y, mb.y);
        m.z = __dadd_rn(m.z, mb.z);
        m.w = __dadd_rn(m.w, mb.w);
        lo = box_min(lo, load_lo(t, ca + 1, tag));
        hi = box_max(hi, load_hi(t, ca + 1, tag));
      }
      double c[3];
      node_com(m.x, m.y, m.z, m.w, c);
      if (t.quad) {
        double S[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
        const double4 pa = t.pred[ca];
        const double cca[3] = {pa.x, pa.y, pa.z};
        add_second_moment(S, t.S64[ca].s, t.mom[ca].x, cca, c);
        if (two) {
          const double4 pb = t.pred[ca + 1];
          const double ccb[3] = {pb.x, pb.y, pb.z};
          add_second_moment(S, t.S64[ca + 1].s, t.mom[ca + 1].x, ccb, c);
        }
        finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, c, lo, hi, true, S);
      } else {
        finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, c, lo, hi, true);
      }
    }
    __syncthreads();
  }
}

__global__ __launch_bounds__(256) void k_permute_f64(const double4* __restrict__ pm_in,
                                                     const double4* __restrict__ vi_in,
                                                     const uint32_t* __restrict__ perm, int64_t n,
                                                     double4* __restrict__ pm_out, double4* __restrict__ vi_out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t p = perm[i];
  pm_out[i] = pm_in[p];
  vi_out[i] = vi_in[p];
}

}  // namespace

void launch_build_fused(const TreeView& t, const float4* leaves, bool keep_all, cudaStream_t s) {
  if (t.L < 1) return;
  const int levels = t.quad ? kFuseLevels - 1 : kFuseLevels;
  const int half = t.quad ? fuse_half<true>() : fuse_half<false>();
  const int top = t.L < levels ? t.L : levels;
  const unsigned grid = unsigned((t.count[1] + half - 1) / half);
  if (t.quad)
    k_build_fused<true, false><<<grid, kFuseThreads, 0, s>>>(t, leaves, top, keep_all);
  else
    k_build_fused<false, false><<<grid, kFuseThreads, 0, s>>>(t, leaves, top, keep_all);
  int from = top + 1;
#if NBODY_UPPER_WIDE > 0
  // the widest upper levels (thousands of nodes) one grid each, the narrow
  // rest in the one-block kernel (same arithmetic, bit-identical records)
  if (!t.quad)
    for (; from <= t.L && from <= top + NBODY_UPPER_WIDE; ++from)
      k_build_level<<<unsigned((t.count[from] + 255) / 256), 256, 0, s>>>(t, from);
#endif
  if (t.L >= from) k_build_upper<false><<<1, 1024, 0, s>>>(t, from);
}

int build_fused_kernels(const TreeView& t) {  // launches of launch_build_fused
  if (t.L < 1) return 0;
  const int levels = t.quad ? kFuseLevels - 1 : kFuseLevels;
  const int top = t.L < levels ? t.L : levels;
  int from = top + 1, k = 1;
  if (!t.quad)
    for (; from <= t.L && from <= top + NBODY_UPPER_WIDE; ++from) ++k;
  return k + (t.L >= from ? 1 : 0);
}

void launch_build_fused_f64(const TreeView& t, bool keep_all, cudaStream_t s) {
  if (t.L < 1) return;
  const int levels = kFuseLevels - 1;  // 512-leaf subtrees (fp64 boxes in shared memory)
  const int half = kFuseHalf / 2;
  const int top = t.L < levels ? t.L : levels;
  const unsigned grid = unsigned((t.count[1] + half - 1) / half);
  k_build_fused<false, true><<<grid, kFuseThreads, 0, s>>>(t, nullptr, top, keep_all);
  if (t.L > top) k_build_upper<true><<<1, 1024, 0, s>>>(t, top + 1);
}

void launch_permute_f64(const double4* pm_in, const double4* vi_in, const uint32_t* perm, int64_t n,
                        double4* pm_out, double4* vi_out, cudaStream_t s) {
  k_permute_f64<<<unsigned((n + 255) / 256), 256, 0, s>>>(pm_in, vi_in, perm, n, pm_out, vi_out);
}

void launch_permute(const float4* pm_in, const float4* vi_in, const uint32_t* perm, int64_t n, float4* pm_out,
                    float4* vi_out, cudaStream_t s) {
  k_permute<<<unsigned((n + 255) / 256), 256, 0, s>>>(pm_in, vi_in, perm, n, pm_out, vi_out);
}

void launch_build(const TreeView& t, const float4* leaves, cudaStream_t s) {
  if (t.L < 1) return;
  k_build_level1<<<unsigned((t.count[1] + 255) / 256), 256, 0, s>>>(t, leaves);
  for (int l = 2; l <= t.L; ++l)
    k_build_level<<<unsigned((t.count[l] + 255) / 256), 256, 0, s>>>(t, l);
}


// Load every kernel of this file now (see preload_all in capi.cu).
void preload_build() {
  touch(k_build_upper<false>);
  touch(k_build_upper<true>);
  touch(k_build_fused<false, false>);
  touch(k_build_fused<false, true>);
  touch(k_build_fused<true, false>);
  touch(k_build_level);
  touch(k_build_level1);
  touch(k_permute);
  touch(k_permute_f64);
}

}  // namespace nb
