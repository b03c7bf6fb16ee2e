/*
 * ccube.h — C ABI of the B200-native C-Cube hot path.
 *
 * C-Cube (Jo, Son, Kim, HPCA'23; /root/reference/PAPER.md cited as P:Lnnn) is a
 * chunk-pipelined tree AllReduce (sum) of data-parallel gradients whose reduce-up
 * and broadcast-down phases overlap per chunk ("C1"), optionally on
 * two complementary trees (fn4 P:L153), plus a gradient queue that lets
 * the next iteration's forward layer l start as soon as the chunks holding its
 * gradients have landed ("C2").
 *
 * Everything on the data path runs in hand-written sm_100a kernels that move data
 * with 128-bit loads/stores into peer GPUs' memory over NVLink 5 / NVSwitch and
 * synchronise through single-writer monotone 64-bit counters (acquire/release,
 * .sys scope).  No NCCL call, no CPU fallback.  The library owns its workspace,
 * peer mappings, trees and Layer-Chunk Table; the caller owns the gradient buffers.
 *
 * Process models (ccube_world_t.nlocal):
 *   nlocal == 1           one process per GPU (torchrun).  Peer memory is mapped
 *                         with CUDA IPC through the caller's allgather callback.
 *   nlocal == world_size  "loopback": one process hosts all P logical ranks on ONE
 *                         GPU; every rank's buffer is local HBM and one kernel
 *                         launch runs the same per-rank kernel body for all ranks.
 *                         Used for single-GPU parity tests and the 1-GPU bench.
 *   Two processes on ONE GPU are refused (their spinning kernels only time-slice)
 *   unless CCUBE_ALLOW_SHARED_GPU=1: the multi-process tests use that to run the
 *   IPC / .sys-scope path on a single GPU.
 *
 * Conventions:
 *   - Collective calls (init, register, allreduce, finalize) must be made by all
 *     ranks in the same order with the same count/dtype/tree kind, as with NCCL.
 *     A mismatch hangs the kernels; the device watchdog (CCUBE_WATCHDOG_MS,
 *     default 10000) then aborts them and the next call returns CCUBE_ERR_TIMEOUT.
 *   - Stream-ordered and asynchronous: allreduce/gradq_wait only enqueue work on
 *     `stream` (a cudaStream_t / CUstream handle; NULL = legacy default stream).
 *   - In place: the reduced result overwrites `buf` ("stored in the same memory
 *     address as where they started reduction").
 *   - Errors: every entry point validates its arguments on the host before any
 *     launch; CUDA failures map to CCUBE_ERR_CUDA; ccube_last_error() returns a
 *     thread-local message describing the last failure.
 */
#ifndef CCUBE_H
#define CCUBE_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define CCUBE_API __attribute__((visibility("default")))
#else
#define CCUBE_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  CCUBE_SUCCESS = 0,
  CCUBE_ERR_INVALID_ARG = -1,
  CCUBE_ERR_NOT_INITIALIZED = -2,
  CCUBE_ERR_ALREADY_INITIALIZED = -3,
  CCUBE_ERR_CUDA = -4,
  CCUBE_ERR_UNSUPPORTED = -5,
  CCUBE_ERR_BOOTSTRAP = -6,
  CCUBE_ERR_TIMEOUT = -7
} ccube_result_t;

/* Tree kind.  SINGLE: one binary tree rooted at rank 0.  DOUBLE: two
 * complementary trees, the second "flipped to invert the nodes and leaves"
 * (fn4 P:L153); chunk c travels on tree c mod 2 (reading R4).
 * ROTATED: the balanced multi-tree set (the NVSwitch form of the
 * topology-aware trees of §IV): P trees, tree t = tree 0 with every
 * rank v renamed (v + t) mod P, chunk c on tree c mod P.  Every rank plays every
 * tree position once, so each GPU's NVLink port carries 2(P-1)/P of the buffer per
 * direction — the bandwidth-optimal load, vs 2 for the double tree at P=8. */
typedef enum {
  CCUBE_TREE_SINGLE = 0,
  CCUBE_TREE_DOUBLE = 1,
  CCUBE_TREE_ROTATED = 2
} ccube_tree_kind_t;

/* Element type.  int32 adds wrap mod 2^32; fp32 adds are IEEE RN (no FMA, no FTZ);
 * bf16 is widened to fp32, added in the fixed order and rounded once (RNE) per
 * tree node (reading R3).  The combine order at a node is own value, then the
 * children's partial sums in ascending rank (reading R2). */
typedef enum { CCUBE_INT32 = 0, CCUBE_FLOAT32 = 1, CCUBE_BFLOAT16 = 2 } ccube_dtype_t;

/* Blocking allgather of `bytes` from every process into recv[p * bytes] (p =
 * process index = rank / nlocal).  Returns 0 on success.  Supplied by the caller
 * (the Python layer wraps a torch.distributed process group).  Called only from
 * inside ccube_init, ccube_register_buffers, ccube_deregister_buffers and
 * ccube_finalize, on the calling thread. */
typedef int (*ccube_allgather_fn)(void *ctx, const void *send, void *recv, size_t bytes);

typedef struct {
  int rank;          /* global rank of the first rank hosted by this process      */
  int nlocal;        /* ranks hosted by this process: 1, or world_size (loopback)  */
  int world_size;    /* P, 1..CCUBE_MAX_RANKS                                       */
  int cuda_device;   /* CUDA device ordinal used by this process                   */
  ccube_allgather_fn allgather;  /* required when nlocal < world_size               */
  void *ctx;                     /* passed back to allgather                        */
} ccube_world_t;

#define CCUBE_MAX_RANKS 8
#define CCUBE_MAX_CHANNELS 128
#define CCUBE_DEFAULT_CHUNK_BYTES (256u * 1024u) /* 256 chunks for 64 MB */

/* ccube_init — collective.  Builds the tree(s), allocates the
 * flag workspace in this GPU's HBM, maps every tree neighbour's workspace (CUDA
 * IPC over NVLink/NVSwitch when nlocal == 1) and zeroes the monotone counters.
 *   chunk_bytes: bytes per pipelined chunk ("the amount of data that is
 *     communicated between neighboring nodes in each step", fn3 P:L88); 0 selects
 *     CCUBE_DEFAULT_CHUNK_BYTES.  Must be a positive multiple of 16 (channel
 *     slices are whole 2 KB units; a chunk shorter than J units leaves the extra
 *     channels an empty slice).
 *   The launch settings read from the environment (CCUBE_CHANNELS, CCUBE_THREADS,
 *   CCUBE_DATAPATH, CCUBE_TRANSPORT, CCUBE_L2_HINTS, CCUBE_SPLIT_CONTROL) are part of
 *   the configuration every rank must share; ccube_init checks them.
 *   (CCUBE_SPLIT_CONTROL: unset = AUTO, one control warp + 7 data warps in the
 *   256-thread CTA geometry on calls of >= 128 chunks, the poll + publish pair
 *   otherwise; 1 / 0 force the pair / the single warp.)
 *   With several processes every tree neighbour on another GPU must be a CUDA peer
 *   (cudaDeviceCanAccessPeer), checked collectively. 
 * Errors: INVALID_ARG (bad world/tree/chunk, ranks disagree on the config or the
 * launch settings),
 * ALREADY_INITIALIZED, UNSUPPORTED (world_size > CCUBE_MAX_RANKS, two processes on
 * one GPU, no peer access), BOOTSTRAP (allgather callback failed), CUDA. */
CCUBE_API ccube_result_t ccube_init(const ccube_world_t *world, ccube_tree_kind_t tree_kind,
                          size_t chunk_bytes);

/* ccube_register_buffers — collective when nlocal < world_size.  Makes the
 * caller's gradient buffer(s) reachable by tree neighbours: the broadcast writes
 * fully reduced chunks straight into each child's buffer, which IS the gradient
 * queue (Fig 9).  Also allocates this rank's receive region
 * (2 x bytes) into which children push their partial sums.
 *   bufs: nlocal device pointers (bufs[i] = buffer of rank world.rank + i), each
 *         16-byte aligned, at least `bytes` long, owned by the caller and kept
 *         alive until ccube_deregister_buffers / ccube_finalize.
 * ccube_allreduce_tree[_local] registers an unseen buffer implicitly (collective). */
CCUBE_API ccube_result_t ccube_register_buffers(void *const *bufs, size_t bytes);
CCUBE_API ccube_result_t ccube_deregister_buffers(void *const *bufs);

/* ccube_allreduce_tree — collective, one-shot: after it completes
 * on `stream`, buf[0..count) on every rank holds the same tree-ordered sum of all
 * ranks' inputs.  Per call the host only validates, looks up the registration,
 * advances the per-tree epoch and launches ONE kernel.  Requires nlocal == 1.
 *   buf:   16-byte aligned device pointer on cuda_device (count * elemsize bytes).
 *   count: elements; 0 is a no-op.  world_size == 1 is a no-op. */
CCUBE_API ccube_result_t ccube_allreduce_tree(void *buf, size_t count, ccube_dtype_t dtype,
                                    void *stream);

/* Same for all nlocal ranks hosted by this process (loopback: bufs[r] for r in
 * 0..P-1, one launch). */
CCUBE_API ccube_result_t ccube_allreduce_tree_local(void *const *bufs, size_t count,
                                          ccube_dtype_t dtype, void *stream);

/* ccube_gradq_set_layers — the Layer-Chunk Table source: element offset
 * at which each layer's gradients end, in forward order (nondecreasing).  Layer l
 * needs the first ceil(layer_end_elems[l] / E) chunks (readings R9, R10). */
CCUBE_API ccube_result_t ccube_gradq_set_layers(const size_t *layer_end_elems, int n_layers);

/* ccube_gradq_wait — enqueue on `stream` a device-side wait until every chunk that
 * holds layer `layer_id`'s gradients (per the most recent allreduce) has landed in
 * this rank's buffer: the "check" of Fig 11 on the Enqueue Semaphore (P:L204,
 * P:L266).  No host synchronisation; the next kernel on `stream` (layer l's update
 * / forward) runs once the wait is satisfied.  The Layer Index Counter is the
 * caller's call order.  Requires nlocal == 1; the _local form takes the local rank
 * index. */
CCUBE_API ccube_result_t ccube_gradq_wait(int layer_id, void *stream);
CCUBE_API ccube_result_t ccube_gradq_wait_local(int local_rank, int layer_id, void *stream);

/* ccube_gradq_set_sgd — fused SGD update at dequeue (the paper gates
 * "update and forward" of layer l on its chunks).  When set, every
 * allreduce also applies, on every rank, w[e] <- w[e] - alpha * g[e] to that rank's
 * fp32 weights, where g is the reduced (summed) gradient — alpha = lr / P gives the
 * averaged SGD step (R14) — as two IEEE-rounded operations, no FMA (reading R18).
 * The step is done by the task that already handles the rank's final gradient (the
 * root's reduce, an interior rank's broadcast, an extra pass at each leaf), and
 * ccube_gradq_wait then opens once the layer's WEIGHTS are updated.
 *   weights: nlocal device pointers (this process's ranks), fp32, 16-byte aligned,
 *            laid out like the gradient buffer (element e <-> element e), at least
 *            `bytes` long, caller-owned; NULL disables the fused update.
 * Errors: NOT_INITIALIZED; UNSUPPORTED for world_size 1 (there is no AllReduce
 * launch to ride on); INVALID_ARG for NULL/misaligned pointers.  While enabled,
 * ccube_allreduce_tree* accepts only CCUBE_FLOAT32 and count * 4 <= bytes. */
CCUBE_API ccube_result_t ccube_gradq_set_sgd(void *const *weights, size_t bytes, float alpha);

/* 1 = C1, the root broadcasts chunk k as soon as it is reduced (default,
 * P:L163); 0 = B, the root broadcasts only after all chunks are reduced (P:L119,
 * the paper's baseline "B").  Values are bitwise identical. */
CCUBE_API ccube_result_t ccube_set_overlap(int on);

/* Settings every rank must share (set_overlap above, set_channels, set_threads,
 * set_datapath, set_transport, gradq_set_sgd on/off): with several processes these
 * setters are COLLECTIVE — every rank calls them in the same order, the value is
 * checked through the allgather callback, and every rank returns INVALID_ARG if
 * any rank passed a different (or invalid) value, leaving the old setting in place.
 *
 * Channels J per tree (CTA slices of every chunk).  0 = auto (CCUBE_CHANNELS env,
 * else the most channels whose CTAs are co-resident on EVERY process — the task
 * count is the maximum over all processes, which depends on every rank's role in
 * every tree, and the capacity the minimum over GPUs — capped at one channel per
 * two 2 KB units of a chunk, or per unit for buffers of >= 16 chunks).  Both ends of
 * an edge therefore always slice chunks alike.  `threads` = data threads per CTA
 * (32..256, multiple of 32; 0 = auto, the default; CCUBE_THREADS env); each CTA
 * adds two control warps.  Smaller CTAs give each thread more registers (two CTAs
 * per SM), which the combines spend on more loads in flight; auto takes 6 data
 * warps when each channel's slice of a chunk holds >= 3 units of 2 KB, else 8. */
CCUBE_API ccube_result_t ccube_set_channels(int channels);
CCUBE_API ccube_result_t ccube_set_threads(int threads);

/* Datapath of the data warps (values are bitwise identical for every choice; all
 * ranks must agree).  LSU: each data warp keeps its own 128-bit loads in flight in
 * registers.  TMA: one data warp streams every source block into a 96 KB
 * shared-memory ring with cp.async.bulk and the other data warps combine from it
 * (needs >= 2 data warps; with one the LSU path runs).  AUTO (default): LSU for every
 * tree kind (round 1 chose TMA for the rotated set; with its leaf-group CTAs LSU is
 * faster there too, measured).  CCUBE_DATAPATH env
 * (0 / 1) sets the initial value.  Errors: NOT_INITIALIZED, INVALID_ARG. */
#define CCUBE_DATAPATH_AUTO (-1)
#define CCUBE_DATAPATH_LSU 0
#define CCUBE_DATAPATH_TMA 1
CCUBE_API ccube_result_t ccube_set_datapath(int datapath);

/* Protocol of one-chunk calls (count * elemsize <= chunk_bytes and <= the LL
 * threshold, CCUBE_LL_MAX_BYTES env, default 256 KiB, at most 1 MiB; no fused
 * update): 1 (default; CCUBE_LL env) = the LL ("low latency") kernel — the same
 * tree-0 fold in the same order (bitwise the same result), but every 8 bytes
 * of payload travel with the call's epoch and the consumer polls the data itself,
 * so a tree hop costs one store-to-load propagation instead of data stores, a
 * fence, a counter store and a counter poll (eq 3's alpha); the LL lines
 * are 2x the payload.  0 = the chunked kernel for every size.  Collective with
 * several processes, like the other settings.  Errors: NOT_INITIALIZED, INVALID_ARG. */
CCUBE_API ccube_result_t ccube_set_protocol(int ll);

/* Edge transport (physical-topology awareness, cf. §IV).  PUSH: a
 * child stores its partial sum into the parent's receive plane (posted NVLink
 * writes, the default across GPUs).  PULL: the child keeps its partial in place
 * in its own buffer and the parent reads it (no receive plane; a leaf moves no
 * data in the reduce phase).  AUTO = PULL for ranks on the same GPU, PUSH across
 * GPUs.  Values are bitwise identical for every choice.  All ranks must agree. */
#define CCUBE_TRANSPORT_AUTO 0
#define CCUBE_TRANSPORT_PUSH 1
#define CCUBE_TRANSPORT_PULL 2
CCUBE_API ccube_result_t ccube_set_transport(int mode);

/* Optional landing trace for gradient-turnaround measurements (Fig 14b):
 * when set, the thread that publishes chunk k of tree t on local rank r also
 * stores %globaltimer (ns) into trace[((r * ntrees + t) * kmax + k) * J + j].
 * NULL disables.  Device pointer of nlocal*ntrees*kmax*J uint64. */
CCUBE_API ccube_result_t ccube_set_trace(uint64_t *trace, size_t kmax);

/* ccube_barrier — collective, device-side: enqueue on `stream` a barrier across all
 * ranks over tree 0's edges (arrive up to the root, release down), using the same
 * monotone counters as the AllReduce; no host synchronisation.  Work enqueued on
 * `stream` after it starts only after every rank has reached it (bench.py puts it
 * before the start event of every timed step).  A no-op when one
 * process hosts every rank (stream order already orders the launch).  Errors:
 * NOT_INITIALIZED, TIMEOUT (an earlier watchdog abort), CUDA. */
CCUBE_API ccube_result_t ccube_barrier(void *stream);

/* ccube_measure_peer_bandwidth — collective (one process per GPU, after
 * ccube_init): the NVLink roofline instrument (SURVEY §8(d) "P2P port-peak
 * microbenchmark").  Times, on the device and after a ccube_barrier, the
 * AllReduce's own cross-GPU data path — 128-bit loads from local HBM, 128-bit
 * stores into a peer's HBM — for `bytes` per destination, best of `iters`.
 *   pair_gbs[i * P + j]: GB/s of rank i's stores into rank j while every rank
 *     stores to its k-th successor at once (k = (j - i) mod P; every port carries one
 *     stream per direction); 0 on the diagonal.
 *   fanout_gbs[m], m = 1..P-1: per-GPU egress GB/s (minimum over ranks) while every
 *     rank stores to its m successors at once; fanout_gbs[0] = 0.
 *   Host arrays of P * P and P doubles, identical on every rank on return.  The
 *   library allocates (and frees) `bytes` + P * `bytes` of scratch and maps every
 *   peer's scratch (not only tree neighbours).
 * Errors: NOT_INITIALIZED; UNSUPPORTED unless nlocal == 1 and world_size >= 2;
 * INVALID_ARG (bytes not a positive multiple of 16, iters < 1, NULL); CUDA. */
CCUBE_API ccube_result_t ccube_measure_peer_bandwidth(size_t bytes, int iters, double *pair_gbs,
                                                      double *fanout_gbs);

/* ccube_plan_launch (host, pure) — the launch geometry the library uses for a call
 * of `bytes` per rank with `channels` (0 = auto) and overlap (1 = C1, 0 = B) when
 * every GPU can hold `cap_ctas` co-resident CTAs: writes the channel count J, the
 * CTAs of the process hosting `rank` (nlocal ranks per process, AUTO transport, no
 * fused update) and the maximum over all processes.  J never depends on `rank`
 * (SURVEY §8(a3)); tests check that for every rank.  Errors: INVALID_ARG. */
CCUBE_API ccube_result_t ccube_plan_launch(int P, ccube_tree_kind_t kind, int nlocal, int rank,
                                           size_t bytes, size_t chunk_bytes, int overlap,
                                           int channels, int cap_ctas, int *channels_out,
                                           int *ctas_out, int *max_ctas_out);

CCUBE_API ccube_result_t ccube_finalize(void);

CCUBE_API const char *ccube_last_error(void);

/* Introspection (host-only, no CUDA needed).  channels/threads are the configured
 * values (0 = auto); last_channels/last_ctas describe the most recent launch. */
typedef struct {
  int initialized, world_size, rank, nlocal, ntrees, channels, threads, overlap, transport;
  size_t chunk_bytes;
  uint64_t epoch_base[2];       /* trees 0 and 1 (ROTATED has P trees) */
  int last_channels, last_ctas;
  int datapath;                 /* configured CCUBE_DATAPATH_* */
  int last_tma;                 /* 1 = the most recent launch ran the TMA datapath */
  int protocol;                 /* configured: 1 = LL for one-chunk calls, 0 = off */
  int last_ll;                  /* 1 = the most recent call ran the LL kernel */
  int last_threads;             /* data threads per CTA of the most recent chunked launch */
} ccube_info_t;
CCUBE_API ccube_result_t ccube_get_info(ccube_info_t *info);

/* The library's own tree builder (host, pure function): parent[v] of tree `tree`
 * (0 for SINGLE, 0..1 for DOUBLE, 0..P-1 for ROTATED) of `kind` for P ranks, -1 at
 * the root. */
CCUBE_API ccube_result_t ccube_tree_parents(int P, ccube_tree_kind_t kind, int tree, int *parent);

/* Placement (reading R19; the NVSwitch form of the paper's detour routes on the
 * DGX-1 cube mesh, §IV: with a direct path between every pair, the
 * topology decision left is which rank hosts which tree position, root included).
 *
 * ccube_set_placement: tree position v of every tree is hosted by rank perm[v]
 * for the NEXT ccube_init (host array of P ints, copied; a permutation of
 * 0..P-1; P must equal that init's world_size).  NULL restores the identity.
 * Children are combined in ascending rank (R2), so a placement can change fp32/
 * bf16 results (never int32's); the oracle takes the same permutation.  Every
 * rank must set the same placement (ccube_init checks it: INVALID_ARG).
 * Errors: ALREADY_INITIALIZED while a communicator exists; INVALID_ARG for a
 * non-permutation or P out of [1, CCUBE_MAX_RANKS].
 *
 * ccube_plan_placement (host, pure): the placement of least cost for a measured
 * peer bandwidth matrix bw[i*P + j] (rank i -> rank j, any unit; <= 0 = no path).
 * Every tree carries 1/T of the buffer up and down each of its edges; the cost
 * of a placement is max over loaded directed pairs of load / bw (the slowest
 * edge sets the pipeline's rate).  Exhaustive over P! placements, ties to the
 * lexicographically smallest (uniform bandwidth -> identity).  Writes P ints to
 * perm.  Errors: INVALID_ARG (NULL pointers, bad kind), UNSUPPORTED for P > 8.
 *
 * ccube_tree_parents_placed: ccube_tree_parents with placement perm (NULL =
 * identity). */
CCUBE_API ccube_result_t ccube_set_placement(const int *perm, int P);
CCUBE_API ccube_result_t ccube_plan_placement(int P, ccube_tree_kind_t kind, const double *bw,
                                              int *perm);
CCUBE_API ccube_result_t ccube_tree_parents_placed(int P, ccube_tree_kind_t kind, int tree,
                                                   const int *perm, int *parent);

#ifdef __cplusplus
}
#endif
#endif /* CCUBE_H */
