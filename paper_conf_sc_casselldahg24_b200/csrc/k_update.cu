// K7 UPDATEPOSITION (Stormer-Verlet; ref [12]) as kick-drift
// leapfrog on half-step velocities [A14]: v_{+1/2} = v_{-1/2} + a dt,
// x_{t+1} = x_t + v_{+1/2} dt (fp32 FMA).  Plus the body packing / id
// scatter helpers of the C ABI.  All HBM bound, one thread per body.
#include <cfloat>

#include "internal.cuh"

namespace nb {
namespace {

__global__ __launch_bounds__(256) void k_leapfrog(const float4* __restrict__ pm_in, const float4* __restrict__ vi_in,
                                                  const float4* __restrict__ acc, int64_t n, float dt,
                                                  float4* __restrict__ pm_out, float4* __restrict__ vi_out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float4 p = pm_in[i], v = vi_in[i];
  const float4 a = acc[i];
  v.x = fmaf(a.x, dt, v.x);
  v.y = fmaf(a.y, dt, v.y);
  v.z = fmaf(a.z, dt, v.z);
  p.x = fmaf(v.x, dt, p.x);
  p.y = fmaf(v.y, dt, p.y);
  p.z = fmaf(v.z, dt, p.z);
  pm_out[i] = p;
  vi_out[i] = v;
}

// K7 with S1 of the next step fused: the same update, grid-
// stride over all n bodies with `gridDim.x` blocks, and each block's min/max
// of the NEW positions into partial[6 * blockIdx.x ..] -- the bounding-box
// partials k_bbox_final reduces at the start of the next pass (Alg. 3,
// P:79-97), so the next pass does not re-read the positions for them.
// Exact (min/max), hence the same box as k_bbox_partial computes.
constexpr int kLFThreads = 512;

__device__ __forceinline__ float wmin(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fminf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float wmax(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

__global__ __launch_bounds__(kLFThreads) void k_leapfrog_bbox(const float4* __restrict__ pm_in,
                                                             const float4* __restrict__ vi_in,
                                                             const float4* __restrict__ acc, int64_t n, float dt,
                                                             float4* __restrict__ pm_out, float4* __restrict__ vi_out,
                                                             float* __restrict__ partial) {
  float lo0 = FLT_MAX, lo1 = FLT_MAX, lo2 = FLT_MAX;
  float hi0 = -FLT_MAX, hi1 = -FLT_MAX, hi2 = -FLT_MAX;
  const int64_t stride = int64_t(gridDim.x) * blockDim.x;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
    float4 p = pm_in[i], v = vi_in[i];
    const float4 a = acc[i];
    v.x = fmaf(a.x, dt, v.x);
    v.y = fmaf(a.y, dt, v.y);
    v.z = fmaf(a.z, dt, v.z);
    p.x = fmaf(v.x, dt, p.x);
    p.y = fmaf(v.y, dt, p.y);
    p.z = fmaf(v.z, dt, p.z);
    pm_out[i] = p;
    vi_out[i] = v;
    lo0 = fminf(lo0, p.x); hi0 = fmaxf(hi0, p.x);
    lo1 = fminf(lo1, p.y); hi1 = fmaxf(hi1, p.y);
    lo2 = fminf(lo2, p.z); hi2 = fmaxf(hi2, p.z);
  }
  __shared__ float sm[kLFThreads / 32][6];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  lo0 = wmin(lo0); lo1 = wmin(lo1); lo2 = wmin(lo2);
  hi0 = wmax(hi0); hi1 = wmax(hi1); hi2 = wmax(hi2);
  if (lane == 0) {
    sm[w][0] = lo0; sm[w][1] = lo1; sm[w][2] = lo2;
    sm[w][3] = hi0; sm[w][4] = hi1; sm[w][5] = hi2;
  }
  __syncthreads();
  if (threadIdx.x < 6) {
    const int c = threadIdx.x;
    float v = sm[0][c];
    for (int k = 1; k < kLFThreads / 32; ++k) v = c < 3 ? fminf(v, sm[k][c]) : fmaxf(v, sm[k][c]);
    partial[6 * blockIdx.x + c] = v;
  }
}

// pos[n][3], vel[n][3], mass[n] -> (x, y, z, m), (vx, vy, vz, id bits).
// *bad |= 1 for a non-finite position/velocity, 2 for a mass <= 0 or
// non-finite [A18].
__global__ __launch_bounds__(256) void k_pack(const float* __restrict__ pos, const float* __restrict__ vel,
                                              const float* __restrict__ mass, int64_t n, float4* __restrict__ pm,
                                              float4* __restrict__ vi, int* __restrict__ bad) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const float x = pos[3 * i], y = pos[3 * i + 1], z = pos[3 * i + 2];
  const float u = vel[3 * i], v = vel[3 * i + 1], w = vel[3 * i + 2];
  const float m = mass[i];
  int flag = 0;
  if (!(isfinite(x) && isfinite(y) && isfinite(z) && isfinite(u) && isfinite(v) && isfinite(w))) flag |= 1;
  if (!(isfinite(m) && m > 0.f)) flag |= 2;
  if (flag) atomicOr(bad, flag);
  pm[i] = make_float4(x, y, z, m);
  vi[i] = make_float4(u, v, w, __int_as_float(int(i)));
}

// nbody_set_state: validate a restored slot-order state in place (the
// checks of k_pack [A18], plus: the ids are a permutation of [0, n) --
// seen[] zeroed by the caller; a second claim of an id is a duplicate).
template <class V4, class S>
__device__ __forceinline__ void check_state(const V4& p, const V4& v, uint32_t id, bool id_ok, int64_t n,
                                            uint32_t* seen, int* bad) {
  int flag = 0;
  if (!(isfinite(p.x) && isfinite(p.y) && isfinite(p.z) && isfinite(v.x) && isfinite(v.y) && isfinite(v.z)))
    flag |= 1;
  if (!(isfinite(p.w) && p.w > S(0))) flag |= 2;
  if (!id_ok || int64_t(id) >= n || atomicExch(seen + id, 1u) != 0u) flag |= 4;
  if (flag) atomicOr(bad, flag);
}

__global__ __launch_bounds__(256) void k_check_state(const float4* __restrict__ pm, const float4* __restrict__ vi,
                                                     int64_t n, uint32_t* __restrict__ seen, int* __restrict__ bad) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const float4 v = vi[i];
  check_state<float4, float>(pm[i], v, uint32_t(__float_as_int(v.w)), true, n, seen, bad);
}

__global__ __launch_bounds__(256) void k_check_state_f64(const double4* __restrict__ pm,
                                                         const double4* __restrict__ vi, int64_t n,
                                                         uint32_t* __restrict__ seen, int* __restrict__ bad) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double4 v = vi[i];
  const bool ok = v.w >= 0.0 && v.w < 4294967296.0 && double(uint32_t(v.w)) == v.w;  // an exact integer id
  check_state<double4, double>(pm[i], v, ok ? uint32_t(v.w) : 0u, ok, n, seen, bad);
}

__global__ __launch_bounds__(256) void k_scatter3(const float4* __restrict__ src, const float4* __restrict__ vi,
                                                  int64_t n, float* __restrict__ out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int64_t id = __float_as_int(vi[i].w);
  const float4 s = src[i];
  out[3 * id] = s.x;
  out[3 * id + 1] = s.y;
  out[3 * id + 2] = s.z;
}

__global__ __launch_bounds__(256) void k_scatter1(const uint32_t* __restrict__ src, const float4* __restrict__ vi,
                                                  int64_t n, uint32_t* __restrict__ out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  out[__float_as_int(vi[i].w)] = src[i];
}

// ---- NEXT-2 FP64 mode: the same helpers on fp64 bodies -------------------
// Leapfrog in fp64 (the oracle's O8 on fp64 state: v + a dt, x + v dt).
__global__ __launch_bounds__(256) void k_leapfrog_f64(const double4* __restrict__ pm_in,
                                                      const double4* __restrict__ vi_in,
                                                      const double4* __restrict__ acc, int64_t n, double dt,
                                                      double4* __restrict__ pm_out, double4* __restrict__ vi_out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double4 p = pm_in[i], v = vi_in[i];
  const double4 a = acc[i];
  v.x = __dadd_rn(v.x, __dmul_rn(a.x, dt));
  v.y = __dadd_rn(v.y, __dmul_rn(a.y, dt));
  v.z = __dadd_rn(v.z, __dmul_rn(a.z, dt));
  p.x = __dadd_rn(p.x, __dmul_rn(v.x, dt));
  p.y = __dadd_rn(p.y, __dmul_rn(v.y, dt));
  p.z = __dadd_rn(p.z, __dmul_rn(v.z, dt));
  pm_out[i] = p;
  vi_out[i] = v;
}

__global__ __launch_bounds__(256) void k_pack_f64(const double* __restrict__ pos, const double* __restrict__ vel,
                                                  const double* __restrict__ mass, int64_t n,
                                                  double4* __restrict__ pm, double4* __restrict__ vi,
                                                  int* __restrict__ bad) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double x = pos[3 * i], y = pos[3 * i + 1], z = pos[3 * i + 2];
  const double u = vel[3 * i], v = vel[3 * i + 1], w = vel[3 * i + 2];
  const double m = mass[i];
  int flag = 0;
  if (!(isfinite(x) && isfinite(y) && isfinite(z) && isfinite(u) && isfinite(v) && isfinite(w))) flag |= 1;
  if (!(isfinite(m) && m > 0.0)) flag |= 2;
  if (flag) atomicOr(bad, flag);
  pm[i] = make_double4(x, y, z, m);
  vi[i] = make_double4(u, v, w, double(i));
}

template <class Out>
__global__ __launch_bounds__(256) void k_scatter3_f64(const double4* __restrict__ src,
                                                      const double4* __restrict__ vi, int64_t n,
                                                      Out* __restrict__ out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int64_t id = int64_t(vi[i].w);
  const double4 s = src[i];
  out[3 * id] = Out(s.x);
  out[3 * id + 1] = Out(s.y);
  out[3 * id + 2] = Out(s.z);
}

__global__ __launch_bounds__(256) void k_scatter1_f64(const uint32_t* __restrict__ src,
                                                      const double4* __restrict__ vi, int64_t n,
                                                      uint32_t* __restrict__ out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  out[int64_t(vi[i].w)] = src[i];
}

__global__ __launch_bounds__(256) void k_fill2(float2* __restrict__ p, int64_t count, float2 v) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i < count) p[i] = v;
}

}  // namespace

void launch_fill_float2(float2* p, int64_t count, float2 v, cudaStream_t s) {
  if (count <= 0) return;
  k_fill2<<<unsigned((count + 255) / 256), 256, 0, s>>>(p, count, v);
}

void launch_leapfrog(const float4* pm_in, const float4* vi_in, const float4* acc, int64_t n, float dt, float4* pm_out,
                     float4* vi_out, cudaStream_t s) {
  if (n <= 0) return;
  k_leapfrog<<<unsigned((n + 255) / 256), 256, 0, s>>>(pm_in, vi_in, acc, n, dt, pm_out, vi_out);
}

void launch_leapfrog_bbox(const float4* pm_in, const float4* vi_in, const float4* acc, int64_t n, float dt,
                          float4* pm_out, float4* vi_out, float* partial, int nparts, cudaStream_t s) {
  if (n <= 0) return;
  k_leapfrog_bbox<<<unsigned(nparts), kLFThreads, 0, s>>>(pm_in, vi_in, acc, n, dt, pm_out, vi_out, partial);
}

void launch_pack_bodies(const float* pos, const float* vel, const float* mass, int64_t n, float4* pm, float4* vi,
                        int* bad, cudaStream_t s) {
  k_pack<<<unsigned((n + 255) / 256), 256, 0, s>>>(pos, vel, mass, n, pm, vi, bad);
}

void launch_check_state(const float4* pm, const float4* vi, int64_t n, uint32_t* seen, int* bad, cudaStream_t s) {
  k_check_state<<<unsigned((n + 255) / 256), 256, 0, s>>>(pm, vi, n, seen, bad);
}

void launch_check_state_f64(const double4* pm, const double4* vi, int64_t n, uint32_t* seen, int* bad,
                            cudaStream_t s) {
  k_check_state_f64<<<unsigned((n + 255) / 256), 256, 0, s>>>(pm, vi, n, seen, bad);
}

void launch_scatter_by_id3(const float4* src, const float4* vi, int64_t n, float* out, cudaStream_t s) {
  if (n <= 0) return;  // a rank may own no slots
  k_scatter3<<<unsigned((n + 255) / 256), 256, 0, s>>>(src, vi, n, out);
}

void launch_scatter_by_id1(const uint32_t* src, const float4* vi, int64_t n, uint32_t* out, cudaStream_t s) {
  if (n <= 0) return;
  k_scatter1<<<unsigned((n + 255) / 256), 256, 0, s>>>(src, vi, n, out);
}

void launch_leapfrog_f64(const double4* pm_in, const double4* vi_in, const double4* acc, int64_t n, double dt,
                         double4* pm_out, double4* vi_out, cudaStream_t s) {
  if (n <= 0) return;
  k_leapfrog_f64<<<unsigned((n + 255) / 256), 256, 0, s>>>(pm_in, vi_in, acc, n, dt, pm_out, vi_out);
}

void launch_pack_bodies_f64(const double* pos, const double* vel, const double* mass, int64_t n, double4* pm,
                            double4* vi, int* bad, cudaStream_t s) {
  k_pack_f64<<<unsigned((n + 255) / 256), 256, 0, s>>>(pos, vel, mass, n, pm, vi, bad);
}

void launch_scatter_by_id3_f64(const double4* src, const double4* vi, int64_t n, double* out, cudaStream_t s) {
  if (n <= 0) return;
  k_scatter3_f64<double><<<unsigned((n + 255) / 256), 256, 0, s>>>(src, vi, n, out);
}

void launch_scatter_by_id3_f64to32(const double4* src, const double4* vi, int64_t n, float* out, cudaStream_t s) {
  if (n <= 0) return;
  k_scatter3_f64<float><<<unsigned((n + 255) / 256), 256, 0, s>>>(src, vi, n, out);
}

void launch_scatter_by_id1_f64(const uint32_t* src, const double4* vi, int64_t n, uint32_t* out, cudaStream_t s) {
  if (n <= 0) return;
  k_scatter1_f64<<<unsigned((n + 255) / 256), 256, 0, s>>>(src, vi, n, out);
}


// Load every kernel of this file now (see preload_all in capi.cu).
void preload_update() {
  touch(k_fill2);
  touch(k_leapfrog);
  touch(k_leapfrog_bbox);
  touch(k_leapfrog_f64);
  touch(k_pack);
  touch(k_pack_f64);
  touch(k_check_state);
  touch(k_check_state_f64);
  touch(k_scatter1);
  touch(k_scatter1_f64);
  touch(k_scatter3);
  touch(k_scatter3_f64<double>);
  touch(k_scatter3_f64<float>);
}

}  // namespace nb
