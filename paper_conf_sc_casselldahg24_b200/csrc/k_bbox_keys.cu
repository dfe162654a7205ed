// K1 CALCULATEBOUNDINGBOX (Alg. 3) and K2 Hilbert keys (P:220,
// Skilling's algorithm, ref [17] P:366).
//
// K1 is an exact fp32 min/max reduction: the result does not depend on the
// reduction order, so it is deterministic and bit-identical to any other
// correct min/max.  K2 quantises in fp64 with explicitly rounded operations
// (no contraction possible in the (x - lo) * inv form) [A9][A16][A17] and
// encodes the cell with Skilling's transform as a 48-state table-driven
// automaton (two levels per shared-memory lookup).  HBM bound: 16 B read per body (K1), 16 B read
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

// Skilling's AxestoTranspose + Gray encoding for 3 axes, read MSB first, as
// a finite-state machine over the levels.  Level q's transformed bits y are
// the raw bits r at level q mapped by the composition T of the exchange /
// inversion steps of the levels above (each acts identically on every lower
// bit position, so T is a map of 3-bit vectors); level q's own step is
//   [y0: invert 0] [y1: invert 0 | else swap 0,1] [y2: invert 0 | else swap 0,2],
// composed onto T for the levels below.  Gray: z = (y0, y1^y0, y2^y1^y0), and
// the output digit is z ^ 111 when the parity p of z2 over the levels above
// is odd (Skilling's t).  The states (T, p) reachable from (identity, 0) are
// 48; the tables are built at compile time:
//   t1[s][r]       = next state << 3 | digit                       (one level)
//   t2[s][a0a1a2]  = state after two levels << 6 | digit_hi << 3 | digit_lo,
// column a0 << 4 | a1 << 2 | a2 with a_i the two bits of axis i (high, low).
// Checked against the oracle's Skilling transform bit for bit (GPU parity
// tests, every b in [1, 21]).
struct HilbertFsm {
  uint16_t t2[48 * 64];
  uint8_t t1[48 * 8];
  int nstates;
};
struct HilbertState {
  uint8_t v[8];  // T as a table of 3-bit vectors
  uint8_t p;
};
constexpr uint8_t hilbert_level_op(uint8_t y, uint8_t v) {
  int v0 = (v >> 2) & 1, v1 = (v >> 1) & 1, v2 = v & 1, t = 0;
  if ((y >> 2) & 1) v0 ^= 1;
  if ((y >> 1) & 1) {
    v0 ^= 1;
  } else {
    t = v0; v0 = v1; v1 = t;
  }
  if (y & 1) {
    v0 ^= 1;
  } else {
    t = v0; v0 = v2; v2 = t;
  }
  return uint8_t((v0 << 2) | (v1 << 1) | v2);
}
constexpr HilbertFsm make_hilbert_fsm() {
  HilbertFsm f{};
  HilbertState st[64]{};
  uint8_t nxt[64][8]{}, out[64][8]{};
  for (int r = 0; r < 8; ++r) st[0].v[r] = uint8_t(r);
  int ns = 1;
  for (int i = 0; i < ns && ns <= 48; ++i) {
    for (int r = 0; r < 8; ++r) {
      const uint8_t y = st[i].v[r];
      const int z0 = (y >> 2) & 1, z1 = ((y >> 1) & 1) ^ z0, z2 = (y & 1) ^ z1;
      out[i][r] = uint8_t(((z0 << 2) | (z1 << 1) | z2) ^ (st[i].p ? 7 : 0));
      HilbertState m{};
      for (int k = 0; k < 8; ++k) m.v[k] = hilbert_level_op(y, st[i].v[k]);
      m.p = uint8_t(st[i].p ^ z2);
      int j = 0;
      for (; j < ns; ++j) {
        bool eq = st[j].p == m.p;
        for (int k = 0; k < 8; ++k) eq = eq && st[j].v[k] == m.v[k];
        if (eq) break;
      }
      if (j == ns && ns < 64) st[ns++] = m;
      nxt[i][r] = uint8_t(j);
    }
  }
  f.nstates = ns;
  for (int i = 0; i < ns && i < 48; ++i) {
    for (int r = 0; r < 8; ++r) f.t1[i * 8 + r] = uint8_t(nxt[i][r] << 3 | out[i][r]);
    for (int c = 0; c < 64; ++c) {
      const int a0 = (c >> 4) & 3, a1 = (c >> 2) & 3, a2 = c & 3;
      const int rh = ((a0 >> 1) << 2) | ((a1 >> 1) << 1) | (a2 >> 1);
      const int rl = ((a0 & 1) << 2) | ((a1 & 1) << 1) | (a2 & 1);
      const int s1 = nxt[i][rh];
      f.t2[i * 64 + c] = uint16_t(nxt[s1][rl] << 6 | out[i][rh] << 3 | out[s1][rl]);
    }
  }
  return f;
}
constexpr HilbertFsm kHilbertFsm = make_hilbert_fsm();
static_assert(kHilbertFsm.nstates == 48, "Skilling's 3-D transform has 48 (T, parity) states");
__device__ const HilbertFsm g_hilbert_fsm = kHilbertFsm;

// The key of cell (x0, x1, x2) at b bits per axis, tables in shared memory.
template <class K, int kB = 0>  // kB > 0: b fixed at compile time (unrolled, constant shifts)
__host__ __device__ __forceinline__ K hilbert_key(uint32_t x0, uint32_t x1, uint32_t x2, int b, const uint16_t* t2,
                                         const uint8_t* t1) {
  uint32_t s = 0;
  K key = 0;
  int q = kB > 0 ? kB : b;
  if (q & 1) {  // odd b: the top level alone
    --q;
    const uint32_t e = t1[((x0 >> q) & 1u) << 2 | ((x1 >> q) & 1u) << 1 | ((x2 >> q) & 1u)];
    key = K(e & 7u);
    s = e >> 3;
  }
#pragma unroll
  while (q > 0) {
    q -= 2;
    const uint32_t c = ((x0 >> q) & 3u) << 4 | ((x1 >> q) & 3u) << 2 | ((x2 >> q) & 3u);
    const uint32_t e = t2[s * 64 + c];
    key = key << 6 | K(e & 63u);
    s = e >> 6;
  }
  return key;
}

constexpr int kKeysThreads = 256;

// Keys, plus the radix-sort digit histograms of every pass (the onesweep
// sort's upfront histogram, fused here so the keys are read only by the
// sort passes).  Grid-stride; per-block shared histograms; a warp whose 32
// keys share a digit adds it once (common for the high digits: the input is
// the previous step's Hilbert order).
// kB, kPasses > 0: the grid resolution and radix passes fixed at compile time
// (the default b = 16: 48-bit keys, 6 passes); 0: read at run time.
template <class K, class V4, int kB = 0, int kPasses = 0>
__global__ __launch_bounds__(kKeysThreads) void k_keys(const V4* __restrict__ pm, int64_t n,
                                                       const GridInfo* __restrict__ gi, K* __restrict__ keys,
                                                       uint32_t* __restrict__ ghist, int passes_rt) {
  const int passes = kPasses > 0 ? kPasses : passes_rt;
  constexpr bool kF64 = sizeof(V4) == 32;  // NEXT-2: fp64 bodies, fp64 box
  __shared__ uint32_t sh[8 * 256];
  __shared__ uint16_t ht2[48 * 64];
  __shared__ uint8_t ht1[48 * 8];
  for (int i = threadIdx.x; i < passes * 256; i += kKeysThreads) sh[i] = 0;
  for (int i = threadIdx.x; i < 48 * 64 / 2; i += kKeysThreads)
    reinterpret_cast<uint32_t*>(ht2)[i] = reinterpret_cast<const uint32_t*>(g_hilbert_fsm.t2)[i];
  for (int i = threadIdx.x; i < 48 * 8; i += kKeysThreads) ht1[i] = g_hilbert_fsm.t1[i];
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
      key = hilbert_key<K, kB>(q0, q1, q2, g.b, ht2, ht1);
      keys[i] = key;
    }
    const uint32_t act = __ballot_sync(0xffffffffu, ok);
#pragma unroll
    for (int ps = 0; ps < (kPasses > 0 ? kPasses : passes); ++ps) {
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
                   int passes, int b, cudaStream_t s) {
  if (b == 16 && passes == 6)  // the default grid
    k_keys<unsigned long long, float4, 16, 6><<<keys_grid(n), kKeysThreads, 0, s>>>(pm, n, g, keys, ghist, passes);
  else
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


// Load every kernel of this file now (see preload_all in capi.cu).
void preload_bbox_keys() {
  touch(k_bbox_final);
  touch(k_bbox_final_f64);
  touch(k_bbox_partial);
  touch(k_bbox_partial_f64);
  touch(k_keys<uint32_t, float4>);
  touch(k_keys<uint32_t, double4>);
  touch(k_keys<unsigned long long, float4, 16, 6>);
  touch(k_keys<unsigned long long, float4>);
  touch(k_keys<unsigned long long, double4>);
}

}  // namespace nb
