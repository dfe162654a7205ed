// K3 HILBERTSORT (Alg. 7): stable LSD radix sort of (key, slot)
// pairs, applied afterwards as a permutation.  [A10] stability makes
// ties keep the current slot order, the same result as std::stable_sort.
//
// Onesweep structure (one upfront histogram pass over all digits, then one
// kernel per 8-bit digit):
//   * tiles of 512 threads x 8 keys = 4096 keys, tile ids from an atomic
//     counter so every tile only ever waits on tiles that already run;
//   * ranking inside a warp by bit-sliced ballots (8 votes per item give the
//     lanes holding the same digit; faster than __match_any_sync here),
//     across the 16 warps of a tile by per-warp shared-memory histograms;
//   * decoupled look-back over per-(tile, digit) status words (2 flag bits +
//     30 count bits, so N < 2^30); a tile publishes its counts before it
//     places its keys in shared memory, and looks back after that (the key
//     registers are free by then);
//   * scatter through shared memory in digit order so that the global stores
//     of a tile are runs of consecutive addresses.
// HBM bound: per pass 2 x (key + 4 B) per body; the upfront histogram reads
// the keys once.
#include <atomic>

#include <cuda/atomic>

#include "internal.cuh"

namespace nb {
namespace {

#ifndef NBODY_SORT_THREADS
#define NBODY_SORT_THREADS 512
#endif
constexpr int kThreads = NBODY_SORT_THREADS;  // >= 256 (one thread per digit)
constexpr int kWarps = kThreads / 32;
#ifndef NBODY_SORT_ITEMS
#define NBODY_SORT_ITEMS 8
#endif
constexpr int kItems = NBODY_SORT_ITEMS;
constexpr int kTile = kThreads * kItems;
constexpr int kRadix = 256;
constexpr uint32_t kFlagAgg = 1u << 30;
constexpr uint32_t kFlagInc = 1u << 31;
constexpr uint32_t kValMask = kFlagAgg - 1u;
#ifndef NBODY_SORT_BALLOT
#define NBODY_SORT_BALLOT 1  // 0: __match_any_sync (0.78 vs 0.67 ms for 6 passes at 1e7)
#endif
#ifndef NBODY_SORT_LOOKBACK
#define NBODY_SORT_LOOKBACK 8
#endif
#ifndef NBODY_SORT_MINB
#define NBODY_SORT_MINB (1024 / NBODY_SORT_THREADS)
#endif
constexpr int kLookback = NBODY_SORT_LOOKBACK;

template <class K>
__device__ __forceinline__ uint32_t digit_of(K k, int shift) {
  return uint32_t(k >> shift) & (kRadix - 1);
}

// Histograms of every digit position in one read of the keys; warp-aggregated
// shared-memory counts (Hilbert keys are heavily skewed in the high digits).
template <class K>
__global__ __launch_bounds__(kThreads) void k_hist(const K* __restrict__ keys, int64_t n, int passes,
                                                   uint32_t* __restrict__ ghist) {
  __shared__ uint32_t sh[8 * kRadix];
  for (int i = threadIdx.x; i < passes * kRadix; i += kThreads) sh[i] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t stride = int64_t(gridDim.x) * kThreads;
  for (int64_t base = int64_t(blockIdx.x) * kThreads + (threadIdx.x & ~31); base < n; base += stride) {
    const int64_t i = base + lane;
    const bool ok = i < n;
    const K k = ok ? keys[i] : K(0);
    for (int p = 0; p < passes; ++p) {
      const uint32_t d = ok ? digit_of(k, 8 * p) : kRadix;
      const uint32_t peers = __match_any_sync(0xffffffffu, d);
      if (ok && lane == __ffs(peers) - 1) atomicAdd(&sh[p * kRadix + d], uint32_t(__popc(peers)));
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < passes * kRadix; i += kThreads)
    if (sh[i]) atomicAdd(&ghist[i], sh[i]);
}

// The global digit offsets of every pass, once per sort: gpre[p][d] =
// sum_{d' < d} ghist[p][d'] (one block; thread d, a loop over the passes).
__global__ __launch_bounds__(kRadix) void k_hist_prefix(const uint32_t* __restrict__ ghist, int passes,
                                                        uint32_t* __restrict__ gpre) {
  __shared__ uint32_t s[kRadix];
  const int d = threadIdx.x;
  for (int p = 0; p < passes; ++p) {
    s[d] = ghist[p * kRadix + d];
    __syncthreads();
    for (int o = 1; o < kRadix; o <<= 1) {  // inclusive scan
      const uint32_t v = d >= o ? s[d - o] : 0u;
      __syncthreads();
      s[d] += v;
      __syncthreads();
    }
    gpre[p * kRadix + d] = s[d] - ghist[p * kRadix + d];
    __syncthreads();
  }
}

// Exclusive scan of v over threads 0..255 (others pass 0); every thread of
// the block must call.  Returns the exclusive prefix for the caller.
__device__ __forceinline__ uint32_t scan256(uint32_t v, uint32_t* s_tmp) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31 && w < kRadix / 32) s_tmp[w] = x;
  __syncthreads();
  uint32_t pre = 0;
  if (w < kRadix / 32)
    for (int j = 0; j < w; ++j) pre += s_tmp[j];
  __syncthreads();
  return pre + x - v;
}

// Design instrumentation (-DNBODY_SORT_PROFILE builds only): SM cycles per
// phase of a tile, summed over tiles (thread 0's clock at the block barriers).
#ifdef NBODY_SORT_PROFILE
__device__ unsigned long long g_sort_prof[8];
#define SORT_T(i) (void)(tid == 0 ? (tp[i] = clock64()) : 0ll)
#else
#define SORT_T(i) ((void)0)
#endif

template <class K, bool kFirst, bool kWriteKeys>
__global__ __launch_bounds__(kThreads, NBODY_SORT_MINB) void k_onesweep(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                       K* __restrict__ kout, uint32_t* __restrict__ vout, int64_t n,
                                                       int shift, const uint32_t* __restrict__ ghist,
                                                       uint32_t* __restrict__ status, uint32_t* __restrict__ tile_ctr) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint32_t* s_whist = reinterpret_cast<uint32_t*>(smem);                  // [kWarps][256]
  K* s_keys = reinterpret_cast<K*>(s_whist + kWarps * kRadix);            // [kTile]
  uint32_t* s_vals = reinterpret_cast<uint32_t*>(s_keys + kTile);         // [kTile]
  __shared__ uint32_t s_dlocal[kRadix], s_dglobal[kRadix], s_tmp[kWarps];
  __shared__ uint32_t s_tile;

  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
#ifdef NBODY_SORT_PROFILE
  long long tp[6];
#endif
  SORT_T(0);
  if (tid == 0) s_tile = atomicAdd(tile_ctr, 1u);
  for (int i = tid; i < kWarps * kRadix; i += kThreads) s_whist[i] = 0;
  __syncthreads();
  SORT_T(1);
  const int64_t tile = s_tile;
  const int64_t base = tile * kTile;

  K k[kItems];
  uint32_t v[kItems], d[kItems], r[kItems];
#pragma unroll
  for (int i = 0; i < kItems; ++i) {
    const int64_t pos = base + w * (32 * kItems) + i * 32 + lane;
    const bool ok = pos < n;
    k[i] = ok ? kin[pos] : K(0);
    v[i] = kFirst ? uint32_t(pos) : (ok ? vin[pos] : 0u);
    d[i] = ok ? digit_of(k[i], shift) : uint32_t(kRadix);
  }
  // Rank inside the warp, in (item, lane) order = position order: stable.
  uint32_t* wh = s_whist + w * kRadix;
  // all matches first (independent, so their latencies overlap) ...
  uint32_t pm[kItems];
#if NBODY_SORT_BALLOT
  // lanes with the same digit by bit-sliced ballots (8 votes per item)
#pragma unroll
  for (int i = 0; i < kItems; ++i) {
    const int64_t rem = n - (base + w * (32 * kItems) + i * 32);  // valid lanes of item i: lane < rem
    uint32_t peers = rem >= 32 ? 0xffffffffu : rem <= 0 ? 0u : (1u << rem) - 1u;
#pragma unroll
    for (int bt = 0; bt < 8; ++bt) {
      const bool on = (d[i] >> bt) & 1u;
      const uint32_t bal = __ballot_sync(0xffffffffu, on);
      peers &= on ? bal : ~bal;
    }
    pm[i] = d[i] < kRadix ? peers : (1u << lane);
  }
#else
#pragma unroll
  for (int i = 0; i < kItems; ++i) pm[i] = __match_any_sync(0xffffffffu, d[i]);
#endif
  // ... then the per-warp digit counters, item by item
#pragma unroll
  for (int i = 0; i < kItems; ++i) {
    const uint32_t peers = pm[i];
    const int leader = __ffs(peers) - 1;
    const uint32_t below = __popc(peers & ((1u << lane) - 1u));
    uint32_t pre = 0;
    if (lane == leader && d[i] < kRadix) {
      pre = wh[d[i]];
      wh[d[i]] = pre + __popc(peers);
    }
    pre = __shfl_sync(0xffffffffu, pre, leader);
    r[i] = pre + below;
    __syncwarp();
  }
  __syncthreads();
  SORT_T(2);

  // Per digit: exclusive prefix over warps (in place) and the tile count.
  uint32_t cnt = 0;
  if (tid < kRadix) {
    for (int j = 0; j < kWarps; ++j) {
      const uint32_t c = s_whist[j * kRadix + tid];
      s_whist[j * kRadix + tid] = cnt;
      cnt += c;
    }
  }
  const uint32_t dl = scan256(tid < kRadix ? cnt : 0u, s_tmp);
  const uint32_t gb = tid < kRadix ? ghist[tid] : 0u;  // this pass's global digit offsets (k_hist_prefix)
  // Publish this tile's digit counts first (successors may look back past
  // it), then place the keys in tile-local digit order in shared memory: that
  // needs only local offsets, and it frees the key registers for the look-back.
  if (tid < kRadix) {
    s_dlocal[tid] = dl;
    cuda::atomic_ref<uint32_t, cuda::thread_scope_device> mine(status[tile * kRadix + tid]);
    mine.store((tile == 0 ? kFlagInc : kFlagAgg) | cnt, cuda::memory_order_relaxed);
  }
  __syncthreads();
  SORT_T(3);
#pragma unroll
  for (int i = 0; i < kItems; ++i) {
    if (d[i] < kRadix) {
      const uint32_t pos = s_dlocal[d[i]] + s_whist[w * kRadix + d[i]] + r[i];
      s_keys[pos] = k[i];
      s_vals[pos] = v[i];
    }
  }
  if (tid < kRadix) {
    if (tile == 0) {
      s_dglobal[tid] = gb;
    } else {
      // Windowed look-back: the status words of up to kLookback predecessors
      // are loaded at once (one L2 round trip), then consumed in order; an
      // unpublished one is re-polled; an inclusive prefix ends the walk.  The
      // window sets how fast the inclusive prefixes advance through the tiles
      // (kLookback tiles per round trip; 8, 16 and 32 measure the same).
      uint32_t excl = 0;
      int64_t p = tile - 1;
      bool done = false;
      while (!done) {
        const int wn = p + 1 < kLookback ? int(p + 1) : kLookback;
        uint32_t sv[kLookback];
#pragma unroll
        for (int i = 0; i < kLookback; ++i)
          if (i < wn) {
            cuda::atomic_ref<uint32_t, cuda::thread_scope_device> o(status[(p - i) * kRadix + tid]);
            sv[i] = o.load(cuda::memory_order_relaxed);
          }
#pragma unroll
        for (int i = 0; i < kLookback; ++i) {
          if (done || i >= wn) continue;
          uint32_t s = sv[i];
          while ((s & ~kValMask) == 0) {  // predecessor not published yet
            cuda::atomic_ref<uint32_t, cuda::thread_scope_device> o(status[(p - i) * kRadix + tid]);
            s = o.load(cuda::memory_order_relaxed);
          }
          excl += s & kValMask;
          if (s & kFlagInc) done = true;
        }
        p -= wn;
      }
      cuda::atomic_ref<uint32_t, cuda::thread_scope_device> mine(status[tile * kRadix + tid]);
      mine.store(kFlagInc | (excl + cnt), cuda::memory_order_relaxed);
      s_dglobal[tid] = gb + excl;
    }
  }
  __syncthreads();
  SORT_T(4);

  // ... and write runs of consecutive global addresses.
  const int valid = int(n - base < kTile ? n - base : int64_t(kTile));
  for (int j = tid; j < valid; j += kThreads) {
    const K key = s_keys[j];
    const uint32_t dd = digit_of(key, shift);
    const int64_t g = int64_t(s_dglobal[dd]) + (j - int64_t(s_dlocal[dd]));
    if (kWriteKeys) kout[g] = key;
    vout[g] = s_vals[j];
  }
#ifdef NBODY_SORT_PROFILE
  __syncthreads();
  SORT_T(5);
  if (tid == 0)
    for (int i = 0; i < 5; ++i) atomicAdd(&g_sort_prof[i], (unsigned long long)(tp[i + 1] - tp[i]));
  if (tid == 0) atomicAdd(&g_sort_prof[5], 1ull);
#endif
}

template <class K>
constexpr size_t dyn_smem() {
  return sizeof(uint32_t) * kWarps * kRadix + sizeof(K) * kTile + sizeof(uint32_t) * kTile;
}

template <class K, bool F, bool W>
void set_attr() {
  cudaFuncSetAttribute(k_onesweep<K, F, W>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn_smem<K>()));
}

template <class K>
void run_sort(const SortPlan& p, void* keys[2], uint32_t* idx[2], cudaStream_t s) {
  // the dynamic shared-memory opt-in is a per-device function attribute
  static std::atomic<uint64_t> attrs_done{0};  // bit d: set on device d
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = uint64_t(1) << (dev & 63);
  if (!(attrs_done.load() & bit)) {
    set_attr<K, true, true>(); set_attr<K, true, false>();
    set_attr<K, false, true>(); set_attr<K, false, false>();
    attrs_done.fetch_or(bit);
  }
  cudaMemsetAsync(p.tile_ctr, 0, sizeof(uint32_t) * 8, s);
  cudaMemsetAsync(p.status, 0, sizeof(uint32_t) * size_t(p.passes) * size_t(p.tiles) * kRadix, s);
  if (!p.hist_ready) {
    cudaMemsetAsync(p.ghist, 0, sizeof(uint32_t) * 8 * kRadix, s);
    const int hb = int(p.tiles < 4 * kNumSMs ? p.tiles : int64_t(4 * kNumSMs));
    k_hist<K><<<hb, kThreads, 0, s>>>(static_cast<const K*>(keys[0]), p.n, p.passes, p.ghist);
  }
  k_hist_prefix<<<1, kRadix, 0, s>>>(p.ghist, p.passes, p.gpre);
  for (int pass = 0; pass < p.passes; ++pass) {
    const int in = pass & 1, out = in ^ 1;
    const K* kin = static_cast<const K*>(keys[in]);
    K* kout = static_cast<K*>(keys[out]);
    const bool first = pass == 0, last = pass == p.passes - 1;
    uint32_t* st = p.status + size_t(pass) * size_t(p.tiles) * kRadix;
    const uint32_t* gh = p.gpre + pass * kRadix;  // exclusive prefix (the kernel's `ghist` argument)
    const unsigned grid = unsigned(p.tiles);
    const size_t sm = dyn_smem<K>();
    if (first && last)
      k_onesweep<K, true, false><<<grid, kThreads, sm, s>>>(kin, idx[in], kout, idx[out], p.n, 8 * pass, gh, st,
                                                          p.tile_ctr + pass);
    else if (first)
      k_onesweep<K, true, true><<<grid, kThreads, sm, s>>>(kin, idx[in], kout, idx[out], p.n, 8 * pass, gh, st,
                                                         p.tile_ctr + pass);
    else if (last)
      k_onesweep<K, false, false><<<grid, kThreads, sm, s>>>(kin, idx[in], kout, idx[out], p.n, 8 * pass, gh, st,
                                                           p.tile_ctr + pass);
    else
      k_onesweep<K, false, true><<<grid, kThreads, sm, s>>>(kin, idx[in], kout, idx[out], p.n, 8 * pass, gh, st,
                                                          p.tile_ctr + pass);
  }
}

}  // namespace

int64_t sort_tiles(int64_t n) { return (n + kTile - 1) / kTile; }

size_t sort_scratch_bytes(int64_t n) {
  return sizeof(uint32_t) * (8 * kRadix + 8 + 8 * kRadix + size_t(8) * size_t(sort_tiles(n)) * kRadix);
}

int launch_radix_sort(const SortPlan& p, void* keys[2], uint32_t* idx[2], cudaStream_t s) {
  if (p.key_bytes == 4)
    run_sort<uint32_t>(p, keys, idx, s);
  else
    run_sort<unsigned long long>(p, keys, idx, s);
  return p.passes & 1;
}


#ifdef NBODY_SORT_PROFILE
extern "C" int nbody_debug_sort_profile(unsigned long long* out) {  // design builds only (not in nbody.h)
  if (cudaMemcpyFromSymbol(out, g_sort_prof, sizeof(unsigned long long) * 6) != cudaSuccess) return -1;
  static const unsigned long long zero[8] = {};
  cudaMemcpyToSymbol(g_sort_prof, zero, sizeof(zero));
  return 6;
}
#endif

// Load every kernel of this file now (see preload_all in capi.cu).
void preload_sort() {
  touch(k_hist<uint32_t>);
  touch(k_hist_prefix);
  touch(k_hist<unsigned long long>);
  touch(k_onesweep<uint32_t, false, false>);
  touch(k_onesweep<uint32_t, false, true>);
  touch(k_onesweep<uint32_t, true, false>);
  touch(k_onesweep<uint32_t, true, true>);
  touch(k_onesweep<unsigned long long, false, false>);
  touch(k_onesweep<unsigned long long, false, true>);
  touch(k_onesweep<unsigned long long, true, false>);
  touch(k_onesweep<unsigned long long, true, true>);
}

}  // namespace nb
