/*
 * nbody.h -- C ABI of the B200-native Hilbert-sorted BVH Barnes-Hut step.
 *
 * Method: Cassell, Deakin, Alpay, Heuveline, Brito Gadeschi, "Efficient
 * Tree-based Parallel Algorithms for N-Body Simulations Using C++ Standard
 * Parallelism", SC'24.  P:NNN below = line NNN of the paper text
 * (/root/reference/PAPER.md); [A#] = a reading of the paper listed in
 * DESIGN.md "Readings".
 *
 * One time step is Alg. 6:
 *   CALCULATEBOUNDINGBOX (Alg. 3) -> HILBERTSORT (Alg. 7,
 *   P:201-212) -> BUILDTREEACCUMULATEMASS (P:218, P:221,
 *   Fig. 4) -> CALCULATEFORCE (Eq. 1
 *   P:72) -> UPDATEPOSITION (Stormer-Verlet).
 * Every stage runs in hand-written sm_100a CUDA kernels of this library.
 *
 * Conventions (all functions):
 *   - G = 1 [A2].  Softened gravity a_i = sum_j m_j r_ij / (|r_ij|^2 + eps^2)^(3/2) [A1].
 *   - Bodies live in "slots".  Slot order is the caller's array order until
 *     the first force pass; afterwards it is the Hilbert order of the last
 *     sort (each step re-sorts the previous step's order).  The body id is
 *     the index in the arrays passed to nbody_set_bodies and travels with
 *     the body.  Functions documented "by id" return arrays indexed by id.
 *   - Pointers to caller buffers may be host (pageable or pinned) or device
 *     pointers of the context's device; the library detects which.  The
 *     caller owns every buffer it passes; the library never keeps a caller
 *     pointer past the call.  Calls that read results synchronise the
 *     context's stream; nbody_step / nbody_compute_accel are asynchronous.
 *   - Not thread-safe per context; one context per (device, stream).
 *   - Every function returns NBODY_OK or a negative status.  No C++
 *     exception or abort crosses the ABI.  After a CUDA failure the context
 *     is in NBODY_ESTATE until nbody_destroy; nbody_last_error() explains.
 */
#ifndef NBODY_B200_H
#define NBODY_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct nbody_ctx nbody_ctx; /* opaque, owned by the library */

typedef enum {
  NBODY_OK = 0,
  NBODY_EINVAL = -1, /* bad argument (null, range, non-finite input)      */
  NBODY_ENOMEM = -2, /* device allocation failed                          */
  NBODY_ECUDA = -3,  /* CUDA error; context now in NBODY_ESTATE           */
  NBODY_ENCCL = -4,  /* NCCL error; context now in NBODY_ESTATE           */
  NBODY_ESTATE = -5  /* call not valid in the current state               */
} nbody_status;

/* Options for nbody_set_option. */
enum {
  /* Hilbert grid bits per axis b [A8]: 0 = the paper's count rule
   * (smallest b with 8^b >= N); 1..21 = fixed b.  Default 16.  Keys hold
   * 3b bits; b <= 10 sorts 32-bit keys, b >= 11 64-bit keys.  Must be set
   * before nbody_set_bodies. */
  NBODY_OPT_KEY_BITS = 1,
  /* cudaStream_t (cast to int64) all work is issued on; 0 = the library's
   * own non-blocking stream (default). */
  NBODY_OPT_STREAM = 2,
  /* 1 = capture one step in a CUDA graph and replay it (default), 0 = plain
   * launches. */
  NBODY_OPT_USE_GRAPH = 3,
  /* CALCULATEFORCE kernel variant: 0 = default (fastest validated),
   * 1 = warp mask-stack walk (per-lane exact lists, no group lists),
   * 2 = the paper's scheme: one thread per body, stackless skip-list DFS
   * (monopole only).  All three give the same interaction
   * lists. */
  NBODY_OPT_TRAVERSAL = 4,
  /* 1 = record CUDA events around each stage of a pass issued by
   * nbody_compute_accel / nbody_step with graphs off; nbody_get_stats then
   * reports the device time of each stage of the last pass.  Default 0. */
  NBODY_OPT_TIMING = 5,
  /* BUILDTREEACCUMULATEMASS kernel variant: 0 = fused 1024-leaf subtrees
   * in shared memory + one block for the top levels (default), 1 = one
   * kernel per level (the paper's level-by-level parallel-for).  Both
   * produce bit-identical records. */
  NBODY_OPT_BUILD = 6,
  /* Tree reuse (NEXT-3(iii); Iwasawa et al., cited at P:320) [A23]: k >= 1;
   * nbody_step re-sorts on steps 0, k, 2k, ... after nbody_set_bodies and
   * otherwise keeps the previous Hilbert order, rebuilding the BVH bottom-up
   * over it at the current positions (no keys, no sort, no permutation).
   * Default 1 (the paper's Alg. 6: sort every step). */
  NBODY_OPT_SORT_EVERY = 7,
  /* Multipole order (NEXT-4; "the algorithms extend to multipoles")
   * [A24]: 1 = monopole (default, the paper's exposition), 2 = monopole +
   * quadrupole: every node also carries its second mass moment about the COM
   * (fp64, parallel-axis theorem) and accepted nodes add the softened
   * quadrupole term.  The opening test, hence every interaction list, is
   * unchanged.  Allocates 80 B per internal node on first use. */
  NBODY_OPT_MULTIPOLE = 8,
  /* NEXT-3(i) cost-weighted Hilbert ranges (P:320 cites
   * load balance as the scale-out concern): 0 = equal slices [A21]
   * (default); 1 = after every force pass the ranks re-split the sorted
   * slots so that each owns about the same number of interactions of that
   * pass (group costs exchanged over peer memory; boundaries multiples of 32
   * slots, slices at most 2 ceil(N/32/G) groups), decided on the device and
   * identical on every rank.  Takes effect only with the fused peer
   * exchange (nbody_attach_peers*); results stay bit-identical to one GPU.
   * nbody_get_partition then reports the range of the last force pass. */
  NBODY_OPT_BALANCE = 9,
  /* NEXT-2 FP64 mode (the paper's own precision: "FP64" throughout, P:272,
   * footnote P:282): 32 (default) or 64.  In mode 64 the state (positions,
   * velocities, masses), the bounding box, the key quantisation, the tree
   * boxes and moments, every interaction and the leapfrog are fp64; the
   * opening decisions are the same fp64 test as in mode 32 (fp32 filters
   * with rigorous bounds decide the clear cases).  Load bodies with
   * nbody_set_bodies64 and read them with the *64 getters (the fp32 getters
   * round).  Setting the option drops the loaded bodies.  Mode 64 needs a
   * single rank (no exchange), monopole order and traversal variant 0
   * (NBODY_EINVAL otherwise); it allocates about 3.7 GB at N = 10^7. */
  NBODY_OPT_PRECISION = 10
};

typedef struct {
  int64_t n;                  /* bodies                                   */
  int key_bits;               /* resolved b                               */
  int levels;                 /* L = ceil(log2 N) levels above the leaves */
  int64_t steps;              /* force passes done since set_bodies       */
  uint64_t interactions;      /* interactions of the last force pass, summed over owned targets */
  float ms_bbox_keys;         /* per-stage device time of the last pass   */
  float ms_sort;              /* (valid only when graphs are off and      */
  float ms_build;             /*  NBODY_OPT_TIMING is on; else 0):        */
  float ms_force;             /*  K1+K2, K3, K4+K5, K6, K7                */
  float ms_update;
  int kernels_per_step;       /* library kernel launches in one step      */
  float lane_util;            /* K6 dense-phase lane utilisation (interacting
                                 lanes / 32 per list slot) since the counters
                                 were last read by nbody_debug_force_stats, in
                                 a -DNBODY_K6_STATS build; -1 otherwise (the
                                 product build carries no counters)        */
} nbody_stats;

/* Library version (major*10000 + minor*100 + patch). */
int nbody_version(void);

/* Make `device` the calling thread's current CUDA device for this library
 * (the library links its own CUDA runtime; callers that select devices
 * through another runtime, e.g. PyTorch, call this before nbody_create). */
nbody_status nbody_select_device(int device);

/* Create a context for n bodies on the current CUDA device.
 *   n in [1, 2^30 - 1] (the sort packs counts in 30 bits); theta >= 0 (opening parameter, accept a node iff
 *   s^2 < theta^2 d^2, [A3]); eps >= 0 (Plummer softening [A1]); dt finite
 *   (leapfrog step [A14]).  All device memory is allocated here (tree
 *   sizes are fixed by N).  *out is set to NULL on failure. */
nbody_status nbody_create(int64_t n, double theta, double eps, double dt, nbody_ctx **out);

/* ---- caller-owned device memory (PyTorch as the allocator) -------------
 * Tree and buffer sizes follow from N alone ("the size of the tree
 * is predetermined by the number of bodies"), so the whole device footprint
 * of a context is known before it exists.  nbody_workspace_bytes returns the
 * bytes of the base workspace (state, keys, sort scratch, tree records,
 * exchange flags) for n bodies on the CURRENT device (the layout depends on
 * its SM count); one layout serves every world <= 256 and every key width
 * b <= 21, so `world` and `key_bits` are only range-checked (0 on a bad
 * argument).  nbody_workspace_bytes_ex adds the optional buffers a context
 * allocates on first use: NBODY_WS_QUAD (quadrupole moments, 80 B per
 * internal node), NBODY_WS_XFER (pipelined-transfer staging, 80 B per body),
 * NBODY_WS_FP64 (the FP64 mode's state and tree). */
enum { NBODY_WS_QUAD = 1, NBODY_WS_XFER = 2, NBODY_WS_FP64 = 4 };
size_t nbody_workspace_bytes(int64_t n, int world, int key_bits);
size_t nbody_workspace_bytes_ex(int64_t n, int world, int key_bits, unsigned features);
/* As nbody_create, but every device buffer of the context is carved, in a
 * fixed order, from dev_workspace[bytes] (a device pointer on the current
 * device, 256-byte aligned, e.g. a torch.empty(bytes, dtype=torch.uint8,
 * device="cuda") tensor): the library allocates no device memory for the
 * context's state.  The caller owns the workspace and must keep it alive
 * until nbody_destroy.  bytes >= nbody_workspace_bytes(n, ...) or
 * NBODY_ENOMEM; optional buffers are taken from the rest of the workspace
 * when first used, and NBODY_ENOMEM is returned then if it does not cover
 * them (size it with nbody_workspace_bytes_ex).  NBODY_EINVAL for a null,
 * misaligned, host or other-device pointer.  Results are bit-identical to
 * a context made by nbody_create.  (nbody_direct_accel, a sampling tool,
 * still takes stream-ordered scratch from the CUDA runtime.) */
nbody_status nbody_create_ws(int64_t n, double theta, double eps, double dt, void *dev_workspace, size_t bytes,
                             nbody_ctx **out);

/* Set an option (see enum).  Returns NBODY_EINVAL for an unknown option or
 * value, NBODY_ESTATE if the option can no longer change. */
nbody_status nbody_set_option(nbody_ctx *ctx, int option, int64_t value);

/* Load the bodies: pos[n][3], vel[n][3] (read as v_{-1/2} [A14]), mass[n],
 * fp32, host or device.  Copies them; resets slot order to array order and
 * ids to array indices.  Masses must be > 0 and finite, positions and
 * velocities finite [A18].  The fp32 interaction forms m (r^2 + eps^2)^(-3/2)
 * in fp32, so units must keep it (for the closest pairs) below ~3e38 [A15];
 * the FP64 mode (NBODY_OPT_PRECISION = 64) has the fp64 range. */
nbody_status nbody_set_bodies(nbody_ctx *ctx, const float *pos, const float *vel, const float *mass);
/* NEXT-2 FP64 mode (NBODY_OPT_PRECISION = 64): as nbody_set_bodies with
 * fp64 pos[n][3], vel[n][3], mass[n] (host or device; copied).
 * NBODY_EINVAL in mode 32, for null pointers or invalid values [A18]. */
nbody_status nbody_set_bodies64(nbody_ctx *ctx, const double *pos, const double *vel, const double *mass);

/* Pipelined host transfers (fp32 mode).  nbody_set_bodies_async does what
 * nbody_set_bodies does, but the copy of pos[n][3], vel[n][3], mass[n]
 * runs on the context's host->device copy stream into one of two device
 * staging buffers, and the packing runs on the context stream after it, so
 * the copy overlaps the steps still queued there.  nbody_get_positions_async
 * enqueues the by-id gather of the current positions on the context
 * stream and the copy into out[n][3] on the device->host copy stream
 * (double-buffered), so the copy overlaps the next steps.  Both return
 * without waiting: the caller keeps the input buffers unchanged and does
 * not read `out` until nbody_sync; host buffers should be pinned for the
 * copies to overlap.  Input validation [A18] is deferred: nbody_sync
 * returns NBODY_EINVAL if any input set since the last sync was invalid
 * (the steps computed from it are then meaningless).  The staging buffers
 * (80 B per body) are allocated on first use.  NBODY_EINVAL in FP64 mode or
 * for null pointers. */
nbody_status nbody_set_bodies_async(nbody_ctx *ctx, const float *pos, const float *vel, const float *mass);
nbody_status nbody_get_positions_async(nbody_ctx *ctx, float *out);

/* Stages 1-5 of Alg. 6 at the current positions (no UPDATEPOSITION):
 * bbox, keys, sort, permute, build, force.  Afterwards slot order is the
 * new Hilbert order and nbody_get_accel returns a(x_t).  Asynchronous. */
nbody_status nbody_compute_accel(nbody_ctx *ctx);

/* nsteps full steps of Alg. 6 (force pass + kick-drift leapfrog
 * v += a dt, x += v dt [A14]).  Asynchronous on the context stream. */
nbody_status nbody_step(nbody_ctx *ctx, int nsteps);

/* Wait for all work issued on the context stream and the copy streams;
 * reports a deferred input error of nbody_set_bodies_async. */
nbody_status nbody_sync(nbody_ctx *ctx);

/* a(x) of the last force pass, out[n][3] by id (fp32). */
nbody_status nbody_get_accel(nbody_ctx *ctx, float *out);

/* Current positions / velocities, out[n][3] by id (fp32). */
nbody_status nbody_get_positions(nbody_ctx *ctx, float *out);
nbody_status nbody_get_velocities(nbody_ctx *ctx, float *out);
/* NEXT-2 FP64 mode: the same outputs in fp64 ([n][3], by body id; host or
 * device out).  NBODY_EINVAL in mode 32. */
nbody_status nbody_get_accel64(nbody_ctx *ctx, double *out);
nbody_status nbody_get_positions64(nbody_ctx *ctx, double *out);
nbody_status nbody_get_velocities64(nbody_ctx *ctx, double *out);

/* Interactions per body of the last force pass, out[n] by id. */
nbody_status nbody_get_interactions(nbody_ctx *ctx, uint32_t *out);

/* Full state in slot order: pos_m[n][4] = (x, y, z, m), vel_id[n][4] =
 * (vx, vy, vz, id reinterpreted as float bits). */
nbody_status nbody_get_state(nbody_ctx *ctx, float *pos_m, float *vel_id);
/* NEXT-2 FP64 mode: the state in slot order, pos_m[n][4] = (x, y, z, m),
 * vel_id[n][4] = (vx, vy, vz, id as an exact integer); either may be NULL.
 * NBODY_EINVAL in mode 32 (and nbody_get_state is NBODY_EINVAL in mode 64). */
nbody_status nbody_get_state64(nbody_ctx *ctx, double *pos_m, double *vel_id);

/* Checkpoint / resume: restore a state exactly as nbody_get_state wrote it
 * -- pos_m[n][4] = (x, y, z, m), vel_id[n][4] = (vx, vy, vz, id as float
 * bits), in slot order, host or device (copied) -- and the step counter
 * `steps` (nbody_stats.steps of the checkpointed context).  Unlike
 * nbody_set_bodies, the slot order and the ids are kept, so the next sort's
 * tie order (the stable sort of Alg. 7 P:201-212 by current slot, [A10]) and
 * the tree-reuse phase (NBODY_OPT_SORT_EVERY, [A23]) are those of the
 * checkpointed run: stepping a restored context is bit-identical to
 * stepping the original.  Every rank passes the same arrays.  NBODY_EINVAL
 * for null pointers, steps < 0, ids that are not a permutation of [0, n),
 * or invalid values [A18] (the context then holds no bodies); in FP64 mode
 * use nbody_set_state64. */
nbody_status nbody_set_state(nbody_ctx *ctx, const float *pos_m, const float *vel_id, int64_t steps);
/* NEXT-2 FP64 mode: as nbody_set_state with the layout of
 * nbody_get_state64 (ids as exact integers in fp64).  NBODY_EINVAL in mode 32. */
nbody_status nbody_set_state64(nbody_ctx *ctx, const double *pos_m, const double *vel_id, int64_t steps);

nbody_status nbody_get_stats(nbody_ctx *ctx, nbody_stats *out);

/* ---- NEXT-1: the paper's All-Pairs baseline, sampled -----------
 * Exact softened direct sum of Eq. 1 [A1] at the current positions,
 * fp64 arithmetic and accumulation, for the bodies with ids[nt] (host or
 * device; host ids are range-checked); out[nt][3] fp64, host or device.
 * Deterministic (fixed-order reduction).  Used to measure Barnes-Hut
 * accuracy against the exact field (config 5). */
nbody_status nbody_direct_accel(nbody_ctx *ctx, const int64_t *ids, int64_t nt, double *out);

/* ---- NEXT-1: the All-Pairs baseline in fp32 at full N ---
 * Softened direct sum of Eq. 1 [A1] at the current positions for the
 * bodies with ids[nt] against ALL n sources, in the fp32 arithmetic of the
 * force kernel's interactions (fp32 differences, FMA, MUFU rsqrt; the
 * target itself adds 0), fp32 partial sums per 2048-source tile and fp64
 * across tiles; out[nt][3] fp64 (host or device).  ids host or device
 * (host ids are range-checked).  Deterministic.  If kernel_ms is not NULL
 * it receives the device time of the all-pairs kernel alone (CUDA events
 * on the context stream) -- the calibration of the FP32 interaction rate
 * the Barnes-Hut force kernel is measured against.  Takes stream-ordered
 * scratch of about 32 B x nt x (source chunks) from the CUDA runtime. */
nbody_status nbody_allpairs_accel(nbody_ctx *ctx, const int64_t *ids, int64_t nt, double *out, float *kernel_ms);

/* ---- multi-GPU: Hilbert-range partition ------------------
 * Every rank holds the whole body state and builds the same tree (all stages
 * up to the tree are deterministic, so the replicas are bit-identical); rank
 * r computes forces and updates only for the sorted slots
 * [r*S, min(N, (r+1)*S)), S = ceil(N / world) rounded up to a multiple of 32
 * [A21].  With a communicator attached, nbody_step ends each step with an
 * NCCL all-gather of the owned body records (the exchange step), so after
 * every step all ranks hold the full updated state; results are
 * bit-identical to one GPU.  nbody_get_accel / nbody_get_interactions are
 * then collective (every rank must call them).  Without a communicator
 * (nbody_set_partition) the context computes its slice only and the caller
 * exchanges slices (nbody_copy_owned) -- the single-GPU emulation the tests
 * use; by-id getters then write only the owned bodies. */

/* The owned slot range of `rank` for n bodies on `world` ranks (host-only,
 * no device needed). */
nbody_status nbody_partition(int64_t n, int rank, int world, int64_t *begin, int64_t *end);
/* 1 if the library was built with NCCL. */
int nbody_has_nccl(void);
/* Write a 128-byte ncclUniqueId (rank 0 creates it, the caller broadcasts it). */
nbody_status nbody_nccl_unique_id(void *out128);
/* Create an NCCL communicator for (rank, world) on the current device and
 * partition the context accordingly.  Collective; call before stepping. */
nbody_status nbody_attach_nccl(nbody_ctx *ctx, const void *unique_id128, int rank, int world);
/* Use an existing NCCL communicator (ncclComm_t passed as void*), e.g. the
 * one torch.distributed's ProcessGroupNCCL created for this device
 * (ProcessGroupNCCL._comm_ptr(), after eager initialisation with device_id):
 * the exchange runs on it instead of a communicator of the library's own.
 * rank and world must equal the communicator's (NBODY_EINVAL otherwise, or
 * if it belongs to another device).  The caller keeps ownership: the
 * communicator must outlive the context and is not destroyed by
 * nbody_destroy.  The library must be linked against the same NCCL as the
 * communicator's creator (build.py links the NCCL that the torch wheel
 * ships).  NBODY_ESTATE if a communicator or peers are already attached;
 * NBODY_ENCCL if the library was built without NCCL. */
nbody_status nbody_attach_comm(nbody_ctx *ctx, void *nccl_comm, int rank, int world);
/* Partition without a communicator (1 <= world <= 256). */
nbody_status nbody_set_partition(nbody_ctx *ctx, int rank, int world);
/* The context's rank, world and owned sorted-slot range [begin, end). */
nbody_status nbody_get_partition(nbody_ctx *ctx, int *rank, int *world, int64_t *begin, int64_t *end);
/* Copy src's owned slice of the body state into dst (same device, same N and
 * world): the exchange step of an emulated partition. */
nbody_status nbody_copy_owned(nbody_ctx *dst, nbody_ctx *src);

/* ---- fused update + exchange over peer memory ------------
 * The alternative to the NCCL all-gather for up to 8 ranks in one NVLink /
 * NVSwitch domain: every rank maps every other rank's state buffers, and the
 * leapfrog kernel (K7 of Alg. 6) stores each updated record of
 * its Hilbert range [A21] straight into the same slot of ALL ranks' state,
 * so the exchange is the update's own stores.  Two device-side barriers per
 * step (flags in each rank's memory, release/acquire at system scope) order
 * the stores against the readers; a barrier that waits > 20 s (a rank that
 * stopped stepping) marks the context failed (NBODY_ESTATE from the next
 * synchronising call).  Results are bit-identical to one GPU.  All ranks
 * must call nbody_step / nbody_compute_accel the same number of times;
 * by-id getters are NOT collective in this mode (they read the peers'
 * forces directly).  Contexts must be destroyed together. */

/* Write this context's 128-byte peer descriptor (a CUDA IPC handle of its
 * device arena plus N and the layout size) for the other ranks. */
nbody_status nbody_peer_handle(nbody_ctx *ctx, void *out128);
/* Map the peers: handles = world descriptors of 128 bytes, indexed by rank
 * (gathered by the caller, e.g. all_gather over torch.distributed), world
 * <= 8, every rank in its own process.  Partitions the context as
 * (rank, world) and selects the fused exchange.  Not with NCCL attached. */
nbody_status nbody_attach_peers(nbody_ctx *ctx, const void *handles128, int rank, int world);
/* The same for `world` contexts of ONE process (ctxs[r] becomes rank r), on
 * one device (single-GPU emulation of the exchange) or on several (peer
 * access is enabled). */
nbody_status nbody_attach_peers_local(nbody_ctx **ctxs, int world);
/* 0 = no exchange (single rank or emulated partition), 1 = NCCL all-gather,
 * 2 = fused peer-memory exchange; -1 for a null context. */
int nbody_exchange_mode(nbody_ctx *ctx);

/* ---- debug views of the last force pass (parity tests) ---------------- */
/* Hilbert keys of the bodies in the slot order BEFORE the last sort:
 * keys[n] as uint64 (3b bits, Skilling's index). */
nbody_status nbody_debug_keys(nbody_ctx *ctx, uint64_t *keys);
/* Sort permutation: sorted slot k <- previous slot perm[k] (stable [A10]). */
nbody_status nbody_debug_perm(nbody_ctx *ctx, uint32_t *perm);
/* Level l in [1, L] of the BVH: *count = ceil(N / 2^l) nodes;
 * pred[count][4] fp64 = (com_x, com_y, com_z, s^2) (the opening-test data,
 * com = sum(m x) / sum(m) in fp64, s = longest AABB side [A3]);
 * rec[count][4] fp32 = ((float)com, (float)M) (the monopole used in the
 * interaction); box[count][6] fp32 = (lo xyz, hi xyz).  Any of pred, rec,
 * box may be NULL; pass all NULL to query *count. */
nbody_status nbody_debug_level(nbody_ctx *ctx, int level, int64_t *count, double *pred, float *rec, float *box);
/* NEXT-2 FP64 mode, after nbody_compute_accel: level l in [1, L]:
 * rec64[count][4] = (com64, M) and box64[count][6] = (lo xyz, hi xyz) in
 * fp64; either may be NULL.  (nbody_debug_level's fp32 box is NBODY_EINVAL
 * in mode 64.) */
nbody_status nbody_debug_level64(nbody_ctx *ctx, int level, int64_t *count, double *rec64, double *box64);

/* NEXT-4: second mass moments about the COM of level l in [1, L] after
 * nbody_compute_accel with NBODY_OPT_MULTIPOLE = 2: S[count][6] fp64 =
 * (xx, yy, zz, xy, xz, yz) [A24]. */
nbody_status nbody_debug_quad(nbody_ctx *ctx, int level, double *S);

/* Design instrumentation of K6: copies up to n event counters of the
 * traversal (summed over all force passes since the last call, then reset)
 * into out and returns how many were written; 0 unless the library was built
 * with -DNBODY_K6_STATS (never in the product build). */
int nbody_debug_force_stats(uint64_t *out, int n);

/* Human-readable description of the last error on this context (never NULL). */
const char *nbody_last_error(const nbody_ctx *ctx);

/* Free all resources.  NULL is a no-op. */
void nbody_destroy(nbody_ctx *ctx);

#ifdef __cplusplus
}
#endif

#endif /* NBODY_B200_H */
