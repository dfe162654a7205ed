// NEXT-1: the paper's All-Pairs baseline (direct
// summation of Eq. 1, softened [A1], G = 1 [A2]) in fp32 at full N --
// the calibration of K6's FP32 roofline: the same interaction arithmetic as
// K6's dense phase (fp32 differences, FMA chain for r^2 + eps^2, MUFU
// rsqrt, m r^-3, three FMA accumulations: 12 FP32-pipe operations = the
// "about 20 flop" of SURVEY 8(d)), with none of the traversal around it.
//
// Tiling (Nyland et al., GPU Gems 3 ch. 31, cited at P:334, re-thought for
// sm_100a): a block stages 2048 sources in shared memory as component-
// interleaved pairs, so one 16-byte broadcast load feeds two sources to the
// packed f32x2 pipe (FADD2/FFMA2/FMUL2: half the issue slots of scalar FP32;
// the FP32 lanes, not issue, then bound the loop); each thread keeps kT
// targets in registers, so a staged pair is used kT times per load.  Sources
// are split into chunks over blockIdx.y for parallelism at small target
// counts; each tile's fp32 partial sums are added into fp64 accumulators
// (bounding the fp32 summation error by one tile's), and the per-chunk
// partials are reduced in a fixed order: results are deterministic.
#include "internal.cuh"

namespace nb {
namespace {

constexpr int kAPThreads = 256;
#ifndef NBODY_AP_T
#define NBODY_AP_T 2
#endif
constexpr int kAPT = NBODY_AP_T;           // targets per thread
#ifndef NBODY_AP_TILE
#define NBODY_AP_TILE 2048
#endif
#ifndef NBODY_AP_UNROLL
#define NBODY_AP_UNROLL 8
#endif
constexpr int kAPTile = NBODY_AP_TILE;    // sources per shared-memory tile (32 KB at 2048)
constexpr int kAPUnroll = NBODY_AP_UNROLL;  // #pragma unroll takes no macros
constexpr int kAPPairs = kAPTile / 2;

struct alignas(16) SrcPair {
  float2 x, y, z, m;
};

__device__ __forceinline__ float rsqrt_fast(float x) {
  float y;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float2 f2(float v) { return make_float2(v, v); }

// Two sources against one target on the packed pipe: a += m r / (r^2 + eps^2)^(3/2),
// r = s - x (nx = -x).  kSoft = false (eps = 0): r^2 = 0 (the target
// itself, a coincident body) adds exactly 0 [A1]; with eps > 0 the target
// itself has r = 0 and adds 0 as well.
template <bool kSoft>
__device__ __forceinline__ void pair2(float2& ax, float2& ay, float2& az, const SrcPair& s, float2 nx, float2 ny,
                                      float2 nz, float2 e2) {
  const float2 dx = __fadd2_rn(s.x, nx), dy = __fadd2_rn(s.y, ny), dz = __fadd2_rn(s.z, nz);
  const float2 r2 = __ffma2_rn(dz, dz, __ffma2_rn(dy, dy, __ffma2_rn(dx, dx, e2)));
  float2 inv = make_float2(rsqrt_fast(r2.x), rsqrt_fast(r2.y));
  if (!kSoft) {
    inv.x = r2.x > 0.f ? inv.x : 0.f;
    inv.y = r2.y > 0.f ? inv.y : 0.f;
  }
  const float2 w = __fmul2_rn(__fmul2_rn(s.m, inv), __fmul2_rn(inv, inv));
  ax = __ffma2_rn(w, dx, ax);
  ay = __ffma2_rn(w, dy, ay);
  az = __ffma2_rn(w, dz, az);
}

// part[c][t] = sum over the sources of chunk c of the softened pair terms for
// target slot tslot[t] (fp32 terms, fp32 per tile, fp64 across tiles).
template <bool kSoft>
__global__ __launch_bounds__(kAPThreads) void k_allpairs32(const float4* __restrict__ pm, int64_t n,
                                                           const uint32_t* __restrict__ tslot, int64_t nt,
                                                           float eps2, int64_t chunk, double4* __restrict__ part) {
  __shared__ SrcPair sp[kAPPairs];
  const int64_t t0 = (int64_t(blockIdx.x) * kAPThreads + threadIdx.x) * kAPT;
  const int64_t c = blockIdx.y;
  const int64_t j0 = c * chunk, j1 = j0 + chunk < n ? j0 + chunk : n;
  float2 nx[kAPT], ny[kAPT], nz[kAPT];
  double ax[kAPT], ay[kAPT], az[kAPT];
#pragma unroll
  for (int i = 0; i < kAPT; ++i) {
    const float4 me = t0 + i < nt ? pm[tslot[t0 + i]] : make_float4(0.f, 0.f, 0.f, 0.f);
    nx[i] = f2(-me.x);
    ny[i] = f2(-me.y);
    nz[i] = f2(-me.z);
    ax[i] = ay[i] = az[i] = 0.0;
  }
  const float2 e2 = f2(eps2);
  for (int64_t base = j0; base < j1; base += kAPTile) {
    __syncthreads();
    for (int k = threadIdx.x; k < kAPPairs; k += kAPThreads) {
      const int64_t j = base + 2 * k;  // zero-mass padding past the chunk end adds exactly 0
      const float4 a = j < j1 ? __ldg(pm + j) : make_float4(0.f, 0.f, 0.f, 0.f);
      const float4 b = j + 1 < j1 ? __ldg(pm + j + 1) : make_float4(0.f, 0.f, 0.f, 0.f);
      SrcPair s;
      s.x = make_float2(a.x, b.x);
      s.y = make_float2(a.y, b.y);
      s.z = make_float2(a.z, b.z);
      s.m = make_float2(a.w, b.w);
      sp[k] = s;
    }
    __syncthreads();
    float2 fx[kAPT], fy[kAPT], fz[kAPT];
#pragma unroll
    for (int i = 0; i < kAPT; ++i) fx[i] = fy[i] = fz[i] = f2(0.f);
    const int np = int(j1 - base >= kAPTile ? kAPPairs : (j1 - base + 1) >> 1);
#pragma unroll kAPUnroll
    for (int p = 0; p < np; ++p) {
      const SrcPair s = sp[p];
#pragma unroll
      for (int i = 0; i < kAPT; ++i) pair2<kSoft>(fx[i], fy[i], fz[i], s, nx[i], ny[i], nz[i], e2);
    }
#pragma unroll
    for (int i = 0; i < kAPT; ++i) {
      ax[i] += double(fx[i].x) + double(fx[i].y);
      ay[i] += double(fy[i].x) + double(fy[i].y);
      az[i] += double(fz[i].x) + double(fz[i].y);
    }
  }
#pragma unroll
  for (int i = 0; i < kAPT; ++i)
    if (t0 + i < nt) part[c * nt + t0 + i] = make_double4(ax[i], ay[i], az[i], 0.0);
}

__global__ void k_allpairs_reduce(const double4* __restrict__ part, int64_t nt, int64_t chunks,
                                  double* __restrict__ out) {
  const int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (t >= nt) return;
  double ax = 0.0, ay = 0.0, az = 0.0;
  for (int64_t c = 0; c < chunks; ++c) {
    const double4 p = part[c * nt + t];
    ax += p.x;
    ay += p.y;
    az += p.z;
  }
  out[3 * t] = ax;
  out[3 * t + 1] = ay;
  out[3 * t + 2] = az;
}

}  // namespace

// Source chunks: about 8 waves of resident blocks over the SMs (the tail of
// the last wave is then at most ~1/8 of the kernel), each chunk a multiple
// of the tile.
int64_t allpairs_chunks(int64_t n, int64_t nt, int nsm) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_allpairs32<true>, kAPThreads, 0) != cudaSuccess ||
      per_sm < 1) {
    cudaGetLastError();
    per_sm = 4;
  }
  const int64_t tblocks = (nt + int64_t(kAPThreads) * kAPT - 1) / (int64_t(kAPThreads) * kAPT);
  const int64_t tiles = (n + kAPTile - 1) / kAPTile;
  int64_t chunks = (8 * int64_t(nsm) * per_sm + tblocks - 1) / tblocks;
  if (chunks > tiles) chunks = tiles;
  if (chunks > 65535) chunks = 65535;
  if (chunks < 1) chunks = 1;
  return chunks;
}

void launch_allpairs32(const float4* pm, int64_t n, const uint32_t* tslot, int64_t nt, float eps2, int64_t chunks,
                       double4* part, double* out, cudaEvent_t ev0, cudaEvent_t ev1, cudaStream_t s) {
  if (nt <= 0) return;
  const int64_t tiles = (n + kAPTile - 1) / kAPTile;
  const int64_t chunk = (tiles + chunks - 1) / chunks * kAPTile;
  dim3 grid(unsigned((nt + int64_t(kAPThreads) * kAPT - 1) / (int64_t(kAPThreads) * kAPT)),
            unsigned((n + chunk - 1) / chunk));
  if (ev0) cudaEventRecord(ev0, s);
  if (eps2 > 0.f)
    k_allpairs32<true><<<grid, kAPThreads, 0, s>>>(pm, n, tslot, nt, eps2, chunk, part);
  else
    k_allpairs32<false><<<grid, kAPThreads, 0, s>>>(pm, n, tslot, nt, eps2, chunk, part);
  if (ev1) cudaEventRecord(ev1, s);
  k_allpairs_reduce<<<unsigned((nt + 255) / 256), 256, 0, s>>>(part, nt, int64_t(grid.y), out);
}


// Load every kernel of this file now (see preload_all in capi.cu).
void preload_allpairs() {
  touch(k_allpairs32<false>);
  touch(k_allpairs32<true>);
  touch(k_allpairs_reduce);
}

}  // namespace nb
