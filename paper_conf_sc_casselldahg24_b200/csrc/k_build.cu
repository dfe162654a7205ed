// K4 permutation gather ("applying it as a permutation afterwards";
// [A11] the whole body state moves) and K5 BUILDTREEACCUMULATEMASS (P:218,
// P:221, Fig. 4; multipoles P:105).
//
// K5 is a parallel-for over the nodes of the next coarser level, level by
// level, reducing the two children (left then right) -- the paper's
// algorithm.  Moments (M, M x) are fp64 sums in that fixed order and the
// boxes exact fp32 min/max, so every node record is bit-identical to the
// oracle's [A12][A13][A16].  Per node it emits the opening-test record
// (com64, s^2) and the fp32 monopole ((float)com64, (float)M) used by K6.
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

// Emit node `node`: the traversal records (pred, rec, rc) always; the build
// moments and box only when `keep` (needed by a parent built in another
// block, or by the debug views).
__device__ __forceinline__ void finish_node(const TreeView& t, int64_t node, double M, double mx, double my, double mz,
                                            float4 lo, float4 hi, bool keep = true) {
  if (keep) {
    t.mom[node] = make_double4(M, mx, my, mz);
    t.blo[node] = lo;
    t.bhi[node] = hi;
  }
  // centre of mass = first moment / mass [A12]
  const double cx = __ddiv_rn(mx, M), cy = __ddiv_rn(my, M), cz = __ddiv_rn(mz, M);
  // [A3] s = longest side of the AABB (fp64 differences of fp32 bounds are exact)
  double s = __dsub_rn(double(hi.x), double(lo.x));
  s = fmax(s, __dsub_rn(double(hi.y), double(lo.y)));
  s = fmax(s, __dsub_rn(double(hi.z), double(lo.z)));
  const double s2 = __dmul_rn(s, s);
  t.pred[node] = make_double4(cx, cy, cz, s2);
  // Filter thresholds on the fp32 squared distance (DESIGN.md "fp32
  // filter"): |d2_fp32 - d^2| <= 1.01e-4 d^2 + A with A = 1e-9 R^2, so
  // d2 > (1 + 2e-4) s^2/theta^2 + A surely accepts and
  // d2 < (1 - 2e-4) s^2/theta^2 - A surely opens.
  float2 rc;
  if (t.th2 > 0.0) {
    const double q = s2 / t.th2;
    const double A = double(t.grid->abs_d2);
    rc.x = __double2float_rd((1.0 - 2e-4) * q - A);
    rc.y = __double2float_ru((1.0 + 2e-4) * q + A);
  } else {  // theta = 0 opens every node
    rc.x = rc.y = __int_as_float(0x7f800000);
  }
  t.rc[node] = rc;
  t.rec[node] = make_float4(__double2float_rn(cx), __double2float_rn(cy), __double2float_rn(cz), __double2float_rn(M));
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
  finish_node(t, t.off[1] + j, M, mx, my, mz, lo, hi);
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
  finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, lo, hi);
}

// Fused build of levels 1..top (top <= 10) over a 1024-leaf subtree per
// block: each level is reduced from the previous one in shared memory (same
// left+right fp64 order, so the records are identical to the level-by-level
// kernels); only the subtree roots (level top) keep moments/boxes in global
// memory unless keep_all (debug views).
constexpr int kFuseLevels = 10;
constexpr int kFuseHalf = 1 << (kFuseLevels - 1);  // level-1 nodes per block
constexpr int kFuseThreads = 256;

__global__ __launch_bounds__(kFuseThreads) void k_build_fused(TreeView t, const float4* __restrict__ leaves, int top,
                                                              bool keep_all) {
  __shared__ double4 s_m[kFuseHalf];
  __shared__ float4 s_lo[kFuseHalf];
  __shared__ float4 s_hi[kFuseHalf];
  const int64_t b = blockIdx.x;
  for (int q = threadIdx.x; q < kFuseHalf; q += kFuseThreads) {
    const int64_t j = b * kFuseHalf + q;
    if (j >= t.count[1]) continue;
    const int64_t a = 2 * j;
    const float4 A = __ldg(leaves + a);
    double M = double(A.w);
    double mx = __dmul_rn(double(A.w), double(A.x));
    double my = __dmul_rn(double(A.w), double(A.y));
    double mz = __dmul_rn(double(A.w), double(A.z));
    float4 lo = make_float4(A.x, A.y, A.z, 0.f), hi = lo;
    if (a + 1 < t.n) {
      const float4 B = __ldg(leaves + a + 1);
      M = __dadd_rn(M, double(B.w));
      mx = __dadd_rn(mx, __dmul_rn(double(B.w), double(B.x)));
      my = __dadd_rn(my, __dmul_rn(double(B.w), double(B.y)));
      mz = __dadd_rn(mz, __dmul_rn(double(B.w), double(B.z)));
      lo.x = fminf(lo.x, B.x); lo.y = fminf(lo.y, B.y); lo.z = fminf(lo.z, B.z);
      hi.x = fmaxf(hi.x, B.x); hi.y = fmaxf(hi.y, B.y); hi.z = fmaxf(hi.z, B.z);
    }
    finish_node(t, t.off[1] + j, M, mx, my, mz, lo, hi, keep_all || top == 1);
    s_m[q] = make_double4(M, mx, my, mz);
    s_lo[q] = lo;
    s_hi[q] = hi;
  }
  __syncthreads();
  for (int l = 2; l <= top; ++l) {
    const int cnt = kFuseHalf >> (l - 1);  // nodes of level l in this block (<= 256)
    const int q = threadIdx.x;
    const int64_t j = b * cnt + q;
    bool have = false;
    double4 m;
    float4 lo, hi;
    if (q < cnt && j < t.count[l]) {
      have = true;
      m = s_m[2 * q];
      lo = s_lo[2 * q];
      hi = s_hi[2 * q];
      if (2 * j + 1 < t.count[l - 1]) {
        const double4 mb = s_m[2 * q + 1];
        const float4 lb = s_lo[2 * q + 1], hb = s_hi[2 * q + 1];
        m.x = __dadd_rn(m.x, mb.x);
        m.y = __dadd_rn(m.y, mb.y);
        m.z = __dadd_rn(m.z, mb.z);
        m.w = __dadd_rn(m.w, mb.w);
        lo.x = fminf(lo.x, lb.x); lo.y = fminf(lo.y, lb.y); lo.z = fminf(lo.z, lb.z);
        hi.x = fmaxf(hi.x, hb.x); hi.y = fmaxf(hi.y, hb.y); hi.z = fmaxf(hi.z, hb.z);
      }
    }
    __syncthreads();
    if (have) {
      s_m[q] = m;
      s_lo[q] = lo;
      s_hi[q] = hi;
      finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, lo, hi, keep_all || l == top);
    }
    __syncthreads();
  }
}

// Levels from..L in one block (the top of the tree is small: ceil(N / 2^l)
// nodes per level); __syncthreads orders the levels.
__global__ __launch_bounds__(1024) void k_build_upper(TreeView t, int from) {
  for (int l = from; l <= t.L; ++l) {
    for (int64_t j = threadIdx.x; j < t.count[l]; j += blockDim.x) {
      const int64_t ca = t.off[l - 1] + 2 * j;
      double4 m = t.mom[ca];
      float4 lo = t.blo[ca], hi = t.bhi[ca];
      if (2 * j + 1 < t.count[l - 1]) {
        const double4 mb = t.mom[ca + 1];
        const float4 lb = t.blo[ca + 1], hb = t.bhi[ca + 1];
        m.x = __dadd_rn(m.x, mb.x);
        m.y = __dadd_rn(m.y, mb.y);
        m.z = __dadd_rn(m.z, mb.z);
        m.w = __dadd_rn(m.w, mb.w);
        lo.x = fminf(lo.x, lb.x); lo.y = fminf(lo.y, lb.y); lo.z = fminf(lo.z, lb.z);
        hi.x = fmaxf(hi.x, hb.x); hi.y = fmaxf(hi.y, hb.y); hi.z = fmaxf(hi.z, hb.z);
      }
      finish_node(t, t.off[l] + j, m.x, m.y, m.z, m.w, lo, hi, true);
    }
    __syncthreads();
  }
}

}  // namespace

void launch_build_fused(const TreeView& t, const float4* leaves, bool keep_all, cudaStream_t s) {
  if (t.L < 1) return;
  const int top = t.L < kFuseLevels ? t.L : kFuseLevels;
  const unsigned grid = unsigned((t.count[1] + kFuseHalf - 1) / kFuseHalf);
  k_build_fused<<<grid, kFuseThreads, 0, s>>>(t, leaves, top, keep_all);
  if (t.L > top) k_build_upper<<<1, 1024, 0, s>>>(t, top + 1);
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

}  // namespace nb
