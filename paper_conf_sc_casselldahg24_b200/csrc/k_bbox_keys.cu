// K1 CALCULATEBOUNDINGBOX (Alg. 3) and K2 Hilbert keys (P:220,
// Skilling's algorithm, ref [17] P:366).
//
// K1 is an exact fp32 min/max reduction: the result does not depend on the
// reduction order, so it is deterministic and bit-identical to any other
// correct min/max.  K2 quantises in fp64 with explicitly rounded operations
// (no contraction possible in the (x - lo) * inv form) [A9][A16][A17] and
// encodes the cell with a branch-free form of Skilling's transpose plus a
// magic-number bit interleave.  HBM bound: 16 B read per body (K1), 16 B read
// + 4/8 B written per body (K2).
#include <float.h>

#include "internal.cuh"

namespace nb {
namespace {

__device__ __forceinline__ float warp_min(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fminf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

constexpr int kBBoxThreads = 512;

// Block-partial min/max of x, y, z over a grid-stride range.
// partial[block][6] = (lo x, lo y, lo z, hi x, hi y, hi z).
__global__ __launch_bounds__(kBBoxThreads) void k_bbox_partial(const float4* __restrict__ pm, int64_t n,
                                                               float* __restrict__ partial) {
  float lo0 = FLT_MAX, lo1 = FLT_MAX, lo2 = FLT_MAX;
  float hi0 = -FLT_MAX, hi1 = -FLT_MAX, hi2 = -FLT_MAX;
  const int64_t stride = int64_t(gridDim.x) * blockDim.x;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
    const float4 p = __ldg(pm + i);
    lo0 = fminf(lo0, p.x); hi0 = fmaxf(hi0, p.x);
    lo1 = fminf(lo1, p.y); hi1 = fmaxf(hi1, p.y);
    lo2 = fminf(lo2, p.z); hi2 = fmaxf(hi2, p.z);
  }
  __shared__ float s[kBBoxThreads / 32][6];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  lo0 = warp_min(lo0); lo1 = warp_min(lo1); lo2 = warp_min(lo2);
  hi0 = warp_max(hi0); hi1 = warp_max(hi1); hi2 = warp_max(hi2);
  if (lane == 0) {
    s[w][0] = lo0; s[w][1] = lo1; s[w][2] = lo2;
    s[w][3] = hi0; s[w][4] = hi1; s[w][5] = hi2;
  }
  __syncthreads();
  if (threadIdx.x < 6) {
    const int c = threadIdx.x;
    float v = s[0][c];
    for (int k = 1; k < kBBoxThreads / 32; ++k) v = c < 3 ? fminf(v, s[k][c]) : fmaxf(v, s[k][c]);
    partial[6 * blockIdx.x + c] = v;
  }
}

// Final reduction of the partials and the grid of the Hilbert keys:
// ext = max_k (hi_k - lo_k) in fp64 (exact for fp32 inputs), inv = 2^b / ext
// (correctly rounded IEEE division), inv = 0 when ext == 0 [A17].
__global__ void k_bbox_final(const float* __restrict__ partial, int nparts, int b, GridInfo* __restrict__ g) {
  __shared__ float s[6];
  const int c = threadIdx.x;
  if (c < 6) {
    float v = partial[c];
    for (int k = 1; k < nparts; ++k) v = c < 3 ? fminf(v, partial[6 * k + c]) : fmaxf(v, partial[6 * k + c]);
    s[c] = v;
  }
  __syncthreads();
  if (c == 0) {
    double ext = 0.0;
    for (int k = 0; k < 3; ++k) {
      g->lo[k] = s[k];
      g->hi[k] = s[3 + k];
      ext = fmax(ext, __dsub_rn(double(s[3 + k]), double(s[k])));
    }
    g->inv = ext > 0.0 ? __ddiv_rn(double(1u << b), ext) : 0.0;
    g->b = b;
    float R = 0.f;
    for (int k = 0; k < 6; ++k) R = fmaxf(R, fabsf(s[k]));
    g->abs_d2 = fmaxf(1e-9f * R * R, 1e-37f);  // larger slack only sends more decisions to fp64
    g->R = R;
  }
}

// NEXT-2 FP64 mode: the same reductions on fp64 bodies (exact min/max).
__device__ __forceinline__ double warp_min_d(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmin(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ double warp_max_d(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

__global__ __launch_bounds__(kBBoxThreads) void k_bbox_partial_f64(const double4* __restrict__ pm, int64_t n,
                                                                   double* __restrict__ partial) {
  double lo[3] = {DBL_MAX, DBL_MAX, DBL_MAX}, hi[3] = {-DBL_MAX, -DBL_MAX, -DBL_MAX};
  const int64_t stride = int64_t(gridDim.x) * blockDim.x;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
    const double4 p = pm[i];
    lo[0] = fmin(lo[0], p.x); hi[0] = fmax(hi[0], p.x);
    lo[1] = fmin(lo[1], p.y); hi[1] = fmax(hi[1], p.y);
    lo[2] = fmin(lo[2], p.z); hi[2] = fmax(hi[2], p.z);
  }
  __shared__ double s[kBBoxThreads / 32][6];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int k = 0; k < 3; ++k) {
    lo[k] = warp_min_d(lo[k]);
    hi[k] = warp_max_d(hi[k]);
  }
  if (lane == 0)
    for (int k = 0; k < 3; ++k) {
      s[w][k] = lo[k];
      s[w][3 + k] = hi[k];
    }
  __syncthreads();
  if (threadIdx.x < 6) {
    const int c = threadIdx.x;
    double v = s[0][c];
    for (int k = 1; k < kBBoxThreads / 32; ++k) v = c < 3 ? fmin(v, s[k][c]) : fmax(v, s[k][c]);
    partial[6 * blockIdx.x + c] = v;
  }
}

// ext = max_k (hi_k - lo_k) rounded in fp64 (the oracle's expression on fp64
// bodies), inv = 2^b / ext; R = max |coordinate| rounded up to fp32; the
// fp32 filter slack covers the extra rounding of x to fp32 (4e-9 R^2 >
// 1e-9 R^2 + the 2uR|d| cross term).
__global__ void k_bbox_final_f64(const double* __restrict__ partial, int nparts, int b, GridInfo* __restrict__ g) {
  __shared__ double s[6];
  const int c = threadIdx.x;
  if (c < 6) {
    double v = partial[c];
    for (int k = 1; k < nparts; ++k) v = c < 3 ? fmin(v, partial[6 * k + c]) : fmax(v, partial[6 * k + c]);
    s[c] = v;
  }
  __syncthreads();
  if (c == 0) {
    double ext = 0.0, R = 0.0;
    for (int k = 0; k < 3; ++k) {
      g->lo64[k] = s[k];
      g->hi64[k] = s[3 + k];
      g->lo[k] = __double2float_rd(s[k]);
      g->hi[k] = __double2float_ru(s[3 + k]);
      ext = fmax(ext, __dsub_rn(s[3 + k], s[k]));
      R = fmax(R, fmax(fabs(s[k]), fabs(s[3 + k])));
    }
    g->inv = ext > 0.0 ? __ddiv_rn(double(1u << b), ext) : 0.0;
    g->b = b;
    const float Rf = __double2float_ru(R);
    g->abs_d2 = fmaxf(4e-9f * Rf * Rf, 1e-37f);
    g->R = Rf;
  }
}

// Spread the low 21 bits of v so that bit q lands at bit 3q.
__device__ __forceinline__ unsigned long long spread3(uint32_t v) {
  unsigned long long x = v & 0x1fffffull;
  x = (x | (x << 32)) & 0x001f00000000ffffull;
  x = (x | (x << 16)) & 0x001f0000ff0000ffull;
  x = (x | (x << 8)) & 0x100f00f00f00f00full;
  x = (x | (x << 4)) & 0x10c30c30c30c30c3ull;
  x = (x | (x << 2)) & 0x1249249249249249ull;
  return x;
}

// Skilling's AxestoTranspose for 3 axes of b bits, written branch-free:
// for each level Q (high to low), axis i either inverts the low bits of X0
// (bit Q of Xi set) or exchanges the low bits of X0 and Xi; then Gray
// encoding.  The index is the transposed bits read MSB first, i.e. bit q of
// X0, X1, X2 at index bits 3q+2, 3q+1, 3q.
__device__ __forceinline__ unsigned long long hilbert3(uint32_t x0, uint32_t x1, uint32_t x2, int b) {
  for (int q = b - 1; q >= 1; --q) {
    const uint32_t Q = 1u << q, P = Q - 1;
    // axis 0: exchange with itself is a no-op, so only the inversion remains
    x0 ^= P & (0u - ((x0 >> q) & 1u));
    uint32_t m = 0u - ((x1 >> q) & 1u);
    x0 ^= P & m;
    uint32_t t = (x0 ^ x1) & P & ~m;
    x0 ^= t; x1 ^= t;
    m = 0u - ((x2 >> q) & 1u);
    x0 ^= P & m;
    t = (x0 ^ x2) & P & ~m;
    x0 ^= t; x2 ^= t;
  }
  x1 ^= x0;
  x2 ^= x1;
  uint32_t t = 0;
  for (int q = b - 1; q >= 1; --q) t ^= ((x2 >> q) & 1u) ? ((1u << q) - 1u) : 0u;
  x0 ^= t; x1 ^= t; x2 ^= t;
  return (spread3(x0) << 2) | (spread3(x1) << 1) | spread3(x2);
}

constexpr int kKeysThreads = 256;

// Keys, plus the radix-sort digit histograms of every pass (the onesweep
// sort's upfront histogram, fused here so the keys are read only by the
// sort passes).  Grid-stride; per-block shared histograms; a warp whose 32
// keys share a digit adds it once (common for the high digits: the input is
// the previous step's Hilbert order).
template <class K, class V4>
__global__ __launch_bounds__(kKeysThreads) void k_keys(const V4* __restrict__ pm, int64_t n,
                                                       const GridInfo* __restrict__ gi, K* __restrict__ keys,
                                                       uint32_t* __restrict__ ghist, int passes) {
  constexpr bool kF64 = sizeof(V4) == 32;  // NEXT-2: fp64 bodies, fp64 box
  __shared__ uint32_t sh[8 * 256];
  for (int i = threadIdx.x; i < passes * 256; i += kKeysThreads) sh[i] = 0;
  __syncthreads();
  const GridInfo g = *gi;
  const uint32_t qmax = (1u << g.b) - 1u;
  const int lane = threadIdx.x & 31;
  const int64_t stride = int64_t(gridDim.x) * kKeysThreads;
  for (int64_t base = int64_t(blockIdx.x) * kKeysThreads + (threadIdx.x & ~31); base < n; base += stride) {
    const int64_t i = base + lane;
    const bool ok = i < n;
    K key = 0;
    if (ok) {
      const V4 p = pm[i];
      const double l0 = kF64 ? g.lo64[0] : double(g.lo[0]), l1 = kF64 ? g.lo64[1] : double(g.lo[1]),
                   l2 = kF64 ? g.lo64[2] : double(g.lo[2]);
      // q_k = min(2^b - 1, floor((x_k - lo_k) * inv)) in fp64; the operand is
      // >= 0, so truncation is the floor.
      const uint32_t q0 = min(qmax, __double2uint_rz(__dmul_rn(__dsub_rn(double(p.x), l0), g.inv)));
      const uint32_t q1 = min(qmax, __double2uint_rz(__dmul_rn(__dsub_rn(double(p.y), l1), g.inv)));
      const uint32_t q2 = min(qmax, __double2uint_rz(__dmul_rn(__dsub_rn(double(p.z), l2), g.inv)));
      key = K(hilbert3(q0, q1, q2, g.b));
      keys[i] = key;
    }
    const uint32_t act = __ballot_sync(0xffffffffu, ok);
    for (int ps = 0; ps < passes; ++ps) {
      const uint32_t d = uint32_t(key >> (8 * ps)) & 255u;
      const uint32_t d0 = __shfl_sync(0xffffffffu, d, 0);
      if (__all_sync(0xffffffffu, !ok || d == d0)) {
        if (lane == 0) atomicAdd(&sh[ps * 256 + d0], uint32_t(__popc(act)));
      } else if (ok) {
        atomicAdd(&sh[ps * 256 + d], 1u);
      }
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < passes * 256; i += kKeysThreads)
    if (sh[i]) atomicAdd(&ghist[i], sh[i]);
}

}  // namespace

void launch_bbox_partial(const float4* pm, int64_t n, float* partial, int nblocks, cudaStream_t s) {
  k_bbox_partial<<<nblocks, kBBoxThreads, 0, s>>>(pm, n, partial);
}

void launch_bbox_final(const float* partial, int nparts, int b, GridInfo* g, cudaStream_t s) {
  k_bbox_final<<<1, 32, 0, s>>>(partial, nparts, b, g);
}

static unsigned keys_grid(int64_t n) {
  const int64_t want = (n + kKeysThreads - 1) / kKeysThreads;
  const int64_t cap = 8 * kNumSMs;  // enough blocks to saturate HBM, few global histogram flushes
  return unsigned(want < cap ? want : cap);
}

void launch_keys32(const float4* pm, int64_t n, const GridInfo* g, uint32_t* keys, uint32_t* ghist, int passes,
                   cudaStream_t s) {
  k_keys<uint32_t><<<keys_grid(n), kKeysThreads, 0, s>>>(pm, n, g, keys, ghist, passes);
}

void launch_keys64(const float4* pm, int64_t n, const GridInfo* g, unsigned long long* keys, uint32_t* ghist,
                   int passes, cudaStream_t s) {
  k_keys<unsigned long long><<<keys_grid(n), kKeysThreads, 0, s>>>(pm, n, g, keys, ghist, passes);
}

void launch_bbox_partial_f64(const double4* pm, int64_t n, double* partial, int nblocks, cudaStream_t s) {
  k_bbox_partial_f64<<<nblocks, kBBoxThreads, 0, s>>>(pm, n, partial);
}

void launch_bbox_final_f64(const double* partial, int nparts, int b, GridInfo* g, cudaStream_t s) {
  k_bbox_final_f64<<<1, 32, 0, s>>>(partial, nparts, b, g);
}

void launch_keys_f64(const double4* pm, int64_t n, const GridInfo* g, void* keys, int key_bytes, uint32_t* ghist,
                     int passes, cudaStream_t s) {
  if (key_bytes == 4)
    k_keys<uint32_t><<<keys_grid(n), kKeysThreads, 0, s>>>(pm, n, g, static_cast<uint32_t*>(keys), ghist, passes);
  else
    k_keys<unsigned long long>
        <<<keys_grid(n), kKeysThreads, 0, s>>>(pm, n, g, static_cast<unsigned long long*>(keys), ghist, passes);
}

}  // namespace nb
