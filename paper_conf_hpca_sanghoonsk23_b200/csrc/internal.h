// internal.h — host/device shared layout of the C-Cube runtime (not part of the ABI).
//
// Workspace per rank (HBM of the GPU that hosts the rank):
//   flags  : kFlagBytes of single-writer monotone u64 counters, one per 64 B line
//            flag(tree, kind, channel) — kind kUpHead0/1: "partial of my k-th chunk
//            is in your receive plane" written by child slot 0/1 into the parent;
//            kind kEnq: the Enqueue Semaphore (Fig 9) written by the
//            parent (or by the root itself) after a fully reduced chunk landed;
//            kind kUpd: with the fused SGD update (NEXT f2), written by this rank's
//            own task once its weights of the chunk are updated (the gate then
//            waits on it instead of kEnq).
//   recv   : per registered buffer, 2 planes x bytes; child slot s of either tree
//            writes its partial sum of chunk c at plane s, element offset c*E
//            (the two trees carry disjoint chunks, so they share the planes).
// Counters are never reset: a call with base B and K_t tree-local chunks drives
// every counter of tree t to B + K_t; waits are ">= B + k + 1" (Fig 11 "check").
#pragma once
#include <stddef.h>
#include <stdint.h>

#ifdef __CUDACC__
#define CCUBE_HD __host__ __device__
#else
#define CCUBE_HD
#endif

namespace ccube {

constexpr int kMaxRanks = 8;
constexpr int kDefaultDataThreads = 192;  // data warps per CTA x 32 (CCUBE_THREADS)
constexpr uint64_t kOneControlMinChunks = 128;  // AUTO control: one control warp from here
constexpr int kMaxChannels = 128;
constexpr int kMaxTrees = 8;  // ROTATED: one tree per rank
constexpr int kMaxChildren = 2;
constexpr int kFlagStride = 64;  // bytes between two counters
constexpr int kFlagStrideU64 = kFlagStride / 8;

// kHalf0/1: progress of the two CTAs of a split task (see Task::halves), written by
// each half for the other.
enum FlagKind {
  kUpHead0 = 0, kUpHead1 = 1, kEnq = 2, kUpd = 3, kHalf0 = 4, kHalf1 = 5, kNumFlagKinds = 6
};

CCUBE_HD inline size_t flag_offset(int tree, int kind, int ch) {
  return ((static_cast<size_t>(tree) * kNumFlagKinds + kind) * kMaxChannels + ch) * kFlagStride;
}
constexpr size_t kFlagBytes =
    static_cast<size_t>(kMaxTrees) * kNumFlagKinds * kMaxChannels * kFlagStride;

// Device-side barrier (ccube_barrier) over tree 0's edges, after the counters:
// "arrive" written by child slot s into its parent, "release" written by the parent
// into the child; single-writer monotone u64 like every other counter.
enum BarrierSlot { kBarArrive0 = 0, kBarArrive1 = 1, kBarRelease = 2, kBarSlots = 3 };
CCUBE_HD inline size_t barrier_offset(int slot) { return kFlagBytes + slot * kFlagStride; }

// Low-latency (LL) protocol for one-chunk messages up to the LL threshold: the data
// carries its own flag.  A 16-byte LL line is {d0, e, d1, e} —
// two 4-byte payload words, each paired with the call's epoch e in one 8-byte word
// (8-byte stores are single-copy atomic), so a reader that sees e twice has the
// line, with no fence, no counter and no separate flag round trip per hop.
// Regions per rank, after the barrier counters: the up-lines of child slot 0 and 1
// (written by the children) and the down-lines (written by the parent), each
// kLLRegionBytes = 2 x kLLMaxBytes.  Plus one u64 per rank counting finished LL CTAs.
constexpr size_t kLLMaxBytes = 1024u * 1024u;   // region capacity; the threshold is
                                                 // CCUBE_LL_MAX_BYTES (default 256 KiB)
constexpr size_t kLLDefaultMaxBytes = 256u * 1024u;
constexpr size_t kLLRegionBytes = 2 * kLLMaxBytes;
enum LLSlot { kLLUp0 = 0, kLLUp1 = 1, kLLDown = 2, kLLSlots = 3 };
constexpr size_t kLLBase = kFlagBytes + 4096;   // barrier counters live below
CCUBE_HD inline size_t ll_offset(int slot) { return kLLBase + slot * kLLRegionBytes; }
constexpr size_t kLLDoneOffset = kLLBase + kLLSlots * kLLRegionBytes;
constexpr size_t kWorkspaceBytes = kLLDoneOffset + kFlagStride;

enum Dtype { kInt32 = 0, kFloat32 = 1, kBFloat16 = 2 };
CCUBE_HD inline int elem_size(int dt) { return dt == kBFloat16 ? 2 : 4; }

// Per (local rank, tree): every pointer the kernel body needs.  "peer" pointers
// are mapped peer memory (CUDA IPC) in multi-process mode and plain local
// pointers in loopback mode; the kernel cannot tell the difference.
//
// Edge transport (physical-topology reading of §IV): an edge whose
// two ranks live on different GPUs is PUSH — the child stores its partial sum into
// the parent's receive plane (posted NVLink writes).  An edge inside one GPU is
// PULL — the child leaves its partial in place in its own buffer and the parent
// reads it from there (no receive plane, no extra copy; a pulled leaf moves no
// data at all in the reduce phase).  Both run the same kernel body; only the
// pointers below differ.
struct TreeParams {
  char *buf;                        // own gradient buffer (= the gradient queue)
  const char *up_src[1 + kMaxChildren];  // own buf, then each child's partial
  char *up_dst;                     // where my partial goes (parent plane / own buf / final)
  char *child_buf[kMaxChildren];    // children's gradient buffers (peer)
  uint64_t *head_in[kMaxChildren];  // own counters written by child slot s (channel 0)
  uint64_t *head_out;               // parent's counter for my slot (peer, channel 0)
  uint64_t *enq;                    // own Enqueue Semaphore (channel 0)
  uint64_t *child_enq[kMaxChildren];// children's Enqueue Semaphores (peer, channel 0)
  int nchild;
  int is_root;
  int leaf_pull;                    // leaf on a PULL edge: publishes all chunks at once
  int self_local;                   // local index of this rank (trace)
  int child_local[kMaxChildren];    // local index of each child, -1 if remote (trace)
  int child_interior[kMaxChildren]; // child has children: its buffer is re-read (DOWN)
  char *w;                          // own fp32 weights (fused SGD, f2), same layout as buf
  uint64_t *upd;                    // own "weights updated" counter (channel 0)
  uint64_t *half_slot[2];           // own progress slots of a split task's halves (channel 0)
};

// UPDATE: a leaf's fused-SGD task (f2) — waits for its chunks to land, then
// w <- w - alpha * g in place (leaves have no DOWN task that reads their result).
enum Role { kRoleUp = 0, kRoleDown = 1, kRoleUpdate = 2 };

enum { kAllChannels = -1 };  // a pulled leaf's single task covers every channel

// A task normally runs on one CTA.  With CCUBE_SPLIT_HEADS=1 the pipeline's head — an
// UP task whose children are all pulled leaves, which reads 3 of the DRAM input
// streams — is split over two CTAs (halves = 2): half h's data warps take every other
// block of the channel's slices, and the channel's counters are published (monotone
// max) once BOTH halves are past a chunk.  Off by default (measured slower).
struct Task {
  int16_t local_rank;
  int16_t tree;
  int16_t role;
  int16_t channel;   // kAllChannels for a pulled leaf (and the leaf-group CTA)
  int16_t half;      // 0, or 1 for the second CTA of a split task; leaf group: the
                     // table index of its first pulled leaf
  int16_t halves;    // 1, or 2 for a split task; leaf group: its number of leaves
  int16_t head;      // 1: an UP task at the pipeline's head (children = pulled leaves)
};

struct LaunchArgs {
  const Task *tasks;
  const TreeParams *params;   // [local_rank * ntrees + tree]
  uint64_t count;             // elements
  uint32_t elems_per_chunk;   // E
  uint32_t pad0;
  uint32_t ntrees;
  uint32_t nchannels;
  uint32_t K[kMaxTrees];      // tree-local chunk counts
  uint64_t base[kMaxTrees];   // counter base of this call per tree
  int overlap;                // 1 = C1, 0 = B
  uint64_t timeout_ns;        // watchdog
  int *err;                   // mapped host word; nonzero = abort
  uint64_t *trace;            // optional landing trace
  uint32_t trace_kmax;
  uint64_t trace_up;          // CCUBE_TRACE_UP: offset (entries) of the reduce-up
                              // hand-off trace in `trace`, 0 = none
  int l2_hints;               // 1 = per-stream L2 eviction priorities (keep re-read data)
  int sgd;                    // 1 = fused SGD update at landing (fp32 only)
  float sgd_alpha;            // w <- w - sgd_alpha * g
  int tma;                    // datapath: 0 = register-staged LSU, 1 = TMA bulk-load ring
  int elem_size;              // bytes per element (2 or 4)
  int split_control;          // 1 = separate poll and publish warps (warps 0, 1)
  int backoff_ns;             // data warps' readiness-spin back-off (0 = spin)
  int debug_nodep;            // CCUBE_DEBUG_NODEP: ignore upstream counters (timing
                              // experiments only — the results are NOT the AllReduce)
};

// Kernel launcher (tree_allreduce.cu).  Returns a cudaError_t as int.
int launch_tree_allreduce(const LaunchArgs &args, int dtype, bool sys_scope, int grid,
                          int threads, void *stream);
constexpr int kMaxGateCounters = 128;
int launch_gate(const uint64_t *const *counters, const uint64_t *targets, int n, int *err,
                uint64_t timeout_ns, bool sys_scope, void *stream);
// ccube_barrier's kernel: one warp per local rank.
struct BarrierRank {
  const uint64_t *arrive[kMaxChildren];  // own arrive counters (written by children)
  uint64_t *parent_arrive;               // parent's arrive counter of my slot, or null
  const uint64_t *release;               // own release counter (written by the parent)
  uint64_t *child_release[kMaxChildren]; // children's release counters
  int nchild;
};
// LL kernel (single-chunk messages): per local rank r, `ctas` CTAs.
struct LLRank {
  char *buf;                              // own gradient buffer
  const char *up_in[kMaxChildren];        // own up-line regions (children write)
  char *up_out;                           // parent's up-line region of my slot, or null
  const char *down_in;                    // own down-line region (parent writes)
  char *down_out[kMaxChildren];           // children's down-line regions
  uint64_t *enq;                          // own Enqueue Semaphore (tree 0, channel 0)
  uint64_t *done;                         // own finished-CTA counter
  int nchild;
};
struct LLArgs {
  LLRank r[kMaxRanks];
  uint64_t count;        // elements
  uint64_t done_base;    // finished-CTA count of every rank before this call
  uint64_t enq_value;    // tree 0's Enqueue Semaphore after this call
  uint32_t epoch;        // LL flag of this call (>= 1)
  int ctas;              // CTAs per rank
  int *err;
  uint64_t timeout_ns;
};
int launch_ll(const LLArgs &args, int dtype, bool sys_scope, int nlocal, int threads,
              void *stream);
int launch_barrier(const BarrierRank *ranks, int n, uint64_t epoch, int *err,
                   uint64_t timeout_ns, bool sys_scope, void *stream);
// ccube_measure_peer_bandwidth's copy: src (local) -> every dst (peer), 128-bit.
int launch_peer_copy(const char *src, char *const *dst, int ndst, size_t bytes, int grid,
                     void *stream);
int query_max_blocks_per_sm(int dtype, bool sys_scope, bool sgd, int threads, int tma,
                            int *blocks);

}  // namespace ccube
