// runtime.cc — host side of the C-Cube library: the C ABI of include/ccube.h.
//
// Per call the host does only argument validation, a registration lookup, the
// chunk arithmetic of a3 (K = ceil(bytes / chunk_bytes), chunk c on tree c mod T)
// and ONE kernel launch; everything on the data path runs on the GPU.
//
// Bootstrap (a2): in multi-process mode (nlocal < world_size) the caller's
// allgather callback carries (i) a config-agreement record, (ii) CUDA IPC handles
// of every rank's flag workspace, and later (iii) handles of registered gradient
// buffers and receive regions.  Only tree neighbours' handles are opened.  This
// replaces the paper's GPUDirect P2P setup with NVLink 5 / NVSwitch peer
// mappings.  In loopback mode (nlocal == world_size) all "peers" are local
// allocations and no IPC is used.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdarg>
#include <climits>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <algorithm>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "ccube.h"
#include "internal.h"
#include "plan.h"
#include "trees.h"

namespace ccube {
namespace {

thread_local std::string g_err;

ccube_result_t fail(ccube_result_t code, const char *fmt, ...) {
  char msg[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(msg, sizeof msg, fmt, ap);
  va_end(ap);
  g_err = msg;
  if (getenv("CCUBE_DEBUG")) fprintf(stderr, "[ccube] error %d: %s\n", code, msg);
  return code;
}

#define CUDA_TRY(expr)                                                                      \
  do {                                                                                      \
    cudaError_t e_ = (expr);                                                                \
    if (e_ != cudaSuccess)                                                                  \
      return fail(CCUBE_ERR_CUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(e_),  \
                  __FILE__, __LINE__);                                                      \
  } while (0)

#define CC_TRY(expr)                         \
  do {                                       \
    ccube_result_t r_ = (expr);              \
    if (r_ != CCUBE_SUCCESS) return r_;      \
  } while (0)

// ---- driver entry points (no link-time dependency on libcuda) ----------------
typedef CUresult (*PFN_batchMemOp)(CUstream, unsigned int, CUstreamBatchMemOpParams *,
                                   unsigned int);
typedef CUresult (*PFN_getAddressRange)(CUdeviceptr *, size_t *, CUdeviceptr);

struct Driver {
  PFN_batchMemOp batchMemOp = nullptr;
  PFN_getAddressRange getAddressRange = nullptr;
  bool loaded = false;
};
Driver g_drv;

void load_driver() {
  if (g_drv.loaded) return;
  g_drv.loaded = true;
  cudaDriverEntryPointQueryResult q;
  void *fn = nullptr;
  if (cudaGetDriverEntryPointByVersion("cuStreamBatchMemOp", &fn, 12000, cudaEnableDefault,
                                       &q) == cudaSuccess &&
      q == cudaDriverEntryPointSuccess)
    g_drv.batchMemOp = reinterpret_cast<PFN_batchMemOp>(fn);
  fn = nullptr;
  if (cudaGetDriverEntryPointByVersion("cuMemGetAddressRange", &fn, 12000, cudaEnableDefault,
                                       &q) == cudaSuccess &&
      q == cudaDriverEntryPointSuccess)
    g_drv.getAddressRange = reinterpret_cast<PFN_getAddressRange>(fn);
}

// ---- IPC bookkeeping ---------------------------------------------------------
struct IpcEntry {
  cudaIpcMemHandle_t handle;
  uint64_t offset;
  uint64_t bytes;
  int32_t valid;
  int32_t pad;
};

struct OpenedHandle {
  void *base;
  int refs;
};
std::map<std::string, OpenedHandle> g_opened;  // key = raw handle bytes

ccube_result_t ipc_open(const cudaIpcMemHandle_t &h, void **base) {
  std::string key(reinterpret_cast<const char *>(&h), sizeof h);
  auto it = g_opened.find(key);
  if (it != g_opened.end()) {
    it->second.refs++;
    *base = it->second.base;
    return CCUBE_SUCCESS;
  }
  void *p = nullptr;
  CUDA_TRY(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
  g_opened[key] = OpenedHandle{p, 1};
  *base = p;
  return CCUBE_SUCCESS;
}

void ipc_close(void *base) {
  for (auto it = g_opened.begin(); it != g_opened.end(); ++it) {
    if (it->second.base == base) {
      if (--it->second.refs == 0) {
        cudaIpcCloseMemHandle(base);
        g_opened.erase(it);
      }
      return;
    }
  }
}

struct Registration {
  std::vector<char *> bufs;       // [nlocal] caller-owned
  size_t bytes = 0;
  size_t plane = 0;               // receive-plane stride: bytes rounded up to 256 B
  std::vector<char *> recv;       // [nlocal] library-owned, 2 * plane each
  std::vector<char *> world_buf;  // [world] usable pointer (local or peer-mapped), or null
  std::vector<char *> world_recv; // [world]
  std::vector<void *> opened;     // IPC bases to close
  TreeParams *d_params = nullptr; // [nlocal * ntrees]
};

struct TaskTable {
  Task *d_tasks = nullptr;
  int n = 0;
};

struct Comm {
  bool init = false;
  bool poisoned = false;
  int world = 0, rank0 = 0, nlocal = 0, device = 0, nproc = 1, proc = 0;
  ccube_allgather_fn allgather = nullptr;
  void *ctx = nullptr;
  int ntrees = 1;
  size_t chunk_bytes = CCUBE_DEFAULT_CHUNK_BYTES;
  Tree trees[kMaxTrees];
  // channels 0 = auto; threads = data threads per CTA: 6 data warps (192) + 2
  // control warps = 256-thread CTAs, 128 registers per thread at two CTAs per SM,
  // 6 vectors per lane and source in flight in the combines (measured)
  int channels = 0, threads = 0, overlap = 1;   // threads 0 = auto
  int tree_kind = CCUBE_TREE_SINGLE;
  uint64_t base[kMaxTrees] = {};
  bool have_call = false;
  uint64_t last_base[kMaxTrees] = {};
  uint32_t last_K[kMaxTrees] = {};
  uint64_t last_E = 0;
  int last_channels = 0;
  int last_ctas = 0;
  int l2_hints = 1;
  int datapath = CCUBE_DATAPATH_AUTO;  // CCUBE_DATAPATH env / ccube_set_datapath
  int last_tma = 0;
  int split_control = -1;             // CCUBE_SPLIT_CONTROL env: 1 poll + publish warps,
                                      // 0 one control warp, -1 auto (per call)
  int backoff_ns = 64;                // CCUBE_BACKOFF_NS env: data warps' spin back-off
  int task_order = 0;                 // CCUBE_TASK_ORDER env: block -> task placement
  int debug_nodep = 0;                // CCUBE_DEBUG_NODEP env: timing experiments only
  bool sgd = false;                 // fused SGD update (f2)
  float sgd_alpha = 0.0f;
  size_t sgd_bytes = 0;
  std::vector<char *> sgd_w;        // [nlocal] weights, gradient-buffer layout
  bool last_sgd = false;
  std::vector<size_t> layer_ends;
  std::vector<char *> flags_local;  // [nlocal]
  std::vector<char *> world_flags;  // [world]
  std::vector<void *> opened_flags;
  int *err_host = nullptr, *err_dev = nullptr;
  std::vector<std::unique_ptr<Registration>> regs;
  std::map<std::pair<int, int>, TaskTable> tasks;  // (channels, overlap * 2 + sgd)
  int transport = CCUBE_TRANSPORT_AUTO;
  bool sys_scope = false;
  uint64_t timeout_ns = 10000ull * 1000000ull;
  int sm_count = 0;
  std::map<std::pair<int, int>, int> max_blocks;  // (dtype*2+sgd + 8*datapath, threads)
  uint64_t *trace = nullptr;
  size_t trace_kmax = 0;
  bool use_memop = true;
  bool gate_flush = false;          // memop waits carry CU_STREAM_WAIT_VALUE_FLUSH
  uint64_t bar_epoch = 0;           // ccube_barrier calls so far
  int split_heads = 0;              // CCUBE_SPLIT_HEADS: the pipeline's head on 2 CTAs/channel
  int ll = 1;                       // CCUBE_LL / ccube_set_protocol: LL for short calls
  uint64_t ll_max = kLLDefaultMaxBytes;  // CCUBE_LL_MAX_BYTES: the LL threshold
  uint32_t ll_epoch = 0;            // LL calls so far (the flag of the next one is +1)
  uint64_t ll_done = 0;             // LL CTAs finished per rank so far
  int last_ll = 0;                  // the most recent call ran the LL kernel
  int last_threads = 0;             // data threads per CTA of the most recent launch
};

Comm g;
std::mutex g_mu;

int env_int(const char *name, int dflt) {
  const char *v = getenv(name);
  return v && *v ? atoi(v) : dflt;
}

bool is_local(int r) { return r >= g.rank0 && r < g.rank0 + g.nlocal; }

bool is_neighbor_of_local(int r) {
  for (int i = 0; i < g.nlocal; ++i) {
    const int v = g.rank0 + i;
    for (int t = 0; t < g.ntrees; ++t) {
      const Tree &tr = g.trees[t];
      if (tr.parent[v] == r) return true;
      for (int s = 0; s < tr.nchild[v]; ++s)
        if (tr.child[v][s] == r) return true;
    }
  }
  return false;
}

ccube_result_t do_allgather(const void *send, void *recv, size_t bytes) {
  if (g.nproc == 1) {
    memcpy(recv, send, bytes);
    return CCUBE_SUCCESS;
  }
  if (!g.allgather) return fail(CCUBE_ERR_BOOTSTRAP, "no allgather callback");
  const int rc = g.allgather(g.ctx, send, recv, bytes);
  if (rc != 0) return fail(CCUBE_ERR_BOOTSTRAP, "allgather callback returned %d", rc);
  return CCUBE_SUCCESS;
}

ccube_result_t check_err_word() {
  if (g.poisoned) return fail(CCUBE_ERR_TIMEOUT, "communicator aborted by an earlier watchdog timeout");
  if (g.err_host && *reinterpret_cast<volatile int *>(g.err_host) != 0) {
    volatile int *e = g.err_host;
    g.poisoned = true;
    const char *what = e[0] == 2   ? "gradient-queue gate"
                       : e[0] == 3 ? "barrier"
                       : e[0] == 4 ? "LL AllReduce"
                                   : "AllReduce";
    return fail(CCUBE_ERR_TIMEOUT,
                "device watchdog fired in the %s kernel (block %d waited for counter >= %d, "
                "saw %d); the communicator must be finalized",
                what, e[1], e[2], e[3]);
  }
  return CCUBE_SUCCESS;
}

// Exchange one pointer per local rank through CUDA IPC (multi-process) and
// produce a usable pointer for every neighbour rank.  In loopback mode the local
// pointers are used directly.
ccube_result_t exchange_ptrs(const std::vector<char *> &local, size_t bytes,
                             std::vector<char *> *world_ptrs, std::vector<void *> *opened,
                             bool every_rank = false) {
  world_ptrs->assign(g.world, nullptr);
  for (int i = 0; i < g.nlocal; ++i) (*world_ptrs)[g.rank0 + i] = local[i];
  if (g.nproc == 1) return CCUBE_SUCCESS;
  load_driver();
  std::vector<IpcEntry> mine(g.nlocal);
  for (int i = 0; i < g.nlocal; ++i) {
    memset(&mine[i], 0, sizeof(IpcEntry));
    CUdeviceptr base = 0;
    size_t sz = 0;
    if (!g_drv.getAddressRange ||
        g_drv.getAddressRange(&base, &sz, reinterpret_cast<CUdeviceptr>(local[i])) != CUDA_SUCCESS)
      return fail(CCUBE_ERR_CUDA, "cuMemGetAddressRange failed for %p", (void *)local[i]);
    CUDA_TRY(cudaIpcGetMemHandle(&mine[i].handle, reinterpret_cast<void *>(base)));
    mine[i].offset = reinterpret_cast<CUdeviceptr>(local[i]) - base;
    mine[i].bytes = bytes;
    mine[i].valid = 1;
  }
  std::vector<IpcEntry> all(static_cast<size_t>(g.nproc) * g.nlocal);
  CC_TRY(do_allgather(mine.data(), all.data(), sizeof(IpcEntry) * g.nlocal));
  for (int r = 0; r < g.world; ++r) {
    if (is_local(r) || (!every_rank && !is_neighbor_of_local(r))) continue;
    const IpcEntry &e = all[r];
    if (!e.valid || e.bytes != bytes)
      return fail(CCUBE_ERR_INVALID_ARG, "rank %d registered %llu bytes, expected %llu", r,
                  (unsigned long long)e.bytes, (unsigned long long)bytes);
    void *b = nullptr;
    CC_TRY(ipc_open(e.handle, &b));
    opened->push_back(b);
    (*world_ptrs)[r] = static_cast<char *>(b) + e.offset;
  }
  return CCUBE_SUCCESS;
}

// PUSH or PULL for the edge child -> parent: PULL inside one
// process (same GPU), PUSH across GPUs, unless forced by ccube_set_transport.
bool edge_is_pull(int child, int parent) {
  return plan_edge_is_pull(g.transport, g.nlocal, child, parent);
}

// The TMA datapath runs only when chosen (AUTO = LSU: round 1's AUTO picked TMA for
// the rotated set, whose slices were long at J = 4; at J = 5 with the leaf-group
// CTAs, LSU measured faster at P = 2 / 4 / 8).  The split of the
// pipeline's head tasks runs on the LSU path with the two control warps, without the
// fused update.
bool want_tma() {
  return g.datapath == CCUBE_DATAPATH_TMA;
}
bool split_heads_now() {
  return g.split_heads && !g.sgd && !want_tma() && g.split_control != 0;
}

PlanIn plan_in(uint64_t bytes) {
  PlanIn in;
  in.split_heads = split_heads_now();
  in.trees = g.trees;
  in.ntrees = g.ntrees;
  in.world = g.world;
  in.nlocal = g.nlocal;
  in.transport = g.transport;
  in.overlap = g.overlap;
  in.sgd = g.sgd;
  in.bytes = bytes;
  in.chunk_bytes = g.chunk_bytes;
  return in;
}

// A setting every rank must share (channels, threads, datapath, transport, overlap,
// the fused update): with several processes the setter is collective and checks
// agreement through the allgather, so every rank accepts or rejects the same value.
// `local` is this rank's own validation of the value; a rank whose value is invalid
// still takes part in the exchange (sending a poison value), so no peer is left
// waiting in the allgather and every rank returns an error.
ccube_result_t agree_setting(const char *what, int64_t value,
                             ccube_result_t local = CCUBE_SUCCESS) {
  const int64_t kBad = INT64_MIN;
  const int64_t mine = local == CCUBE_SUCCESS ? value : kBad;
  if (g.nproc > 1) {
    std::vector<int64_t> all(g.nproc);
    const std::string saved = g_err;
    CC_TRY(do_allgather(&mine, all.data(), sizeof mine));
    if (local != CCUBE_SUCCESS) {
      g_err = saved;
      return local;
    }
    for (int p = 0; p < g.nproc; ++p)
      if (all[p] != mine)
        return fail(CCUBE_ERR_INVALID_ARG, "ranks disagree on %s (process %d: %s%lld, here: %lld)",
                    what, p, all[p] == kBad ? "invalid " : "", (long long)all[p], (long long)mine);
  } else if (local != CCUBE_SUCCESS) {
    return local;
  }
  return CCUBE_SUCCESS;
}

bool needs_recv_planes() {
  for (int i = 0; i < g.nlocal; ++i) {
    const int r = g.rank0 + i;
    for (int t = 0; t < g.ntrees; ++t)
      for (int s = 0; s < g.trees[t].nchild[r]; ++s)
        if (!edge_is_pull(g.trees[t].child[r][s], r)) return true;
  }
  return false;
}

ccube_result_t build_params(Registration *R) {
  std::vector<TreeParams> hp(static_cast<size_t>(g.nlocal) * g.ntrees);
  for (int i = 0; i < g.nlocal; ++i) {
    const int r = g.rank0 + i;
    for (int t = 0; t < g.ntrees; ++t) {
      const Tree &tr = g.trees[t];
      TreeParams &p = hp[static_cast<size_t>(i) * g.ntrees + t];
      memset(&p, 0, sizeof p);
      p.buf = R->bufs[i];
      p.up_src[0] = R->bufs[i];
      p.nchild = tr.nchild[r];
      p.is_root = tr.parent[r] < 0;
      p.self_local = i;
      char *fl = g.flags_local[i];
      for (int s = 0; s < kMaxChildren; ++s) {
        p.head_in[s] = reinterpret_cast<uint64_t *>(fl + flag_offset(t, kUpHead0 + s, 0));
        p.child_local[s] = -1;
      }
      p.enq = reinterpret_cast<uint64_t *>(fl + flag_offset(t, kEnq, 0));
      p.upd = reinterpret_cast<uint64_t *>(fl + flag_offset(t, kUpd, 0));
      for (int h = 0; h < 2; ++h)
        p.half_slot[h] = reinterpret_cast<uint64_t *>(fl + flag_offset(t, kHalf0 + h, 0));
      p.w = g.sgd ? g.sgd_w[i] : nullptr;
      const int par = tr.parent[r];
      if (par < 0) {
        p.up_dst = R->bufs[i];  // the root's combine is final
      } else {
        const int slot = child_slot(tr, par, r);
        if (!g.world_flags[par])
          return fail(CCUBE_ERR_BOOTSTRAP, "parent %d of rank %d not mapped", par, r);
        p.head_out =
            reinterpret_cast<uint64_t *>(g.world_flags[par] + flag_offset(t, kUpHead0 + slot, 0));
        if (edge_is_pull(r, par)) {
          p.up_dst = R->bufs[i];  // partial stays in place; the parent reads it here
          p.leaf_pull = tr.nchild[r] == 0;
        } else {
          if (!R->world_recv[par])
            return fail(CCUBE_ERR_BOOTSTRAP, "receive plane of parent %d not mapped", par);
          p.up_dst = R->world_recv[par] + static_cast<size_t>(slot) * R->plane;
        }
      }
      for (int s = 0; s < tr.nchild[r]; ++s) {
        const int c = tr.child[r][s];
        if (!R->world_buf[c] || !g.world_flags[c])
          return fail(CCUBE_ERR_BOOTSTRAP, "child %d of rank %d not mapped", c, r);
        p.child_buf[s] = R->world_buf[c];
        p.child_enq[s] = reinterpret_cast<uint64_t *>(g.world_flags[c] + flag_offset(t, kEnq, 0));
        p.child_local[s] = is_local(c) ? c - g.rank0 : -1;
        p.child_interior[s] = tr.nchild[c] > 0;
        if (edge_is_pull(c, r)) {
          p.up_src[1 + s] = R->world_buf[c];
        } else {
          if (!R->recv[i]) return fail(CCUBE_ERR_BOOTSTRAP, "receive plane missing");
          p.up_src[1 + s] = R->recv[i] + static_cast<size_t>(s) * R->plane;
        }
      }
    }
  }
  if (!R->d_params) CUDA_TRY(cudaMalloc(&R->d_params, sizeof(TreeParams) * hp.size()));
  CUDA_TRY(cudaMemcpy(R->d_params, hp.data(), sizeof(TreeParams) * hp.size(),
                      cudaMemcpyHostToDevice));
  return CCUBE_SUCCESS;
}

void free_registration(Registration *R) {
  for (void *b : R->opened) ipc_close(b);
  R->opened.clear();
  for (char *p : R->recv)
    if (p) cudaFree(p);
  R->recv.clear();
  if (R->d_params) cudaFree(R->d_params);
  R->d_params = nullptr;
}

ccube_result_t do_register(void *const *bufs, size_t bytes, Registration **out) {
  if (!bufs) return fail(CCUBE_ERR_INVALID_ARG, "bufs is NULL");
  if (bytes == 0) return fail(CCUBE_ERR_INVALID_ARG, "bytes == 0");
  for (int i = 0; i < g.nlocal; ++i) {
    if (!bufs[i]) return fail(CCUBE_ERR_INVALID_ARG, "bufs[%d] is NULL", i);
    if (reinterpret_cast<uintptr_t>(bufs[i]) % 16)
      return fail(CCUBE_ERR_INVALID_ARG, "bufs[%d] = %p is not 16-byte aligned", i, bufs[i]);
  }
  std::unique_ptr<Registration> R(new Registration);
  R->bytes = bytes;
  R->plane = (bytes + 255) & ~static_cast<size_t>(255);
  for (int i = 0; i < g.nlocal; ++i) R->bufs.push_back(static_cast<char *>(bufs[i]));
  R->recv.assign(g.nlocal, nullptr);
  // receive planes exist only for PUSH edges; multi-process communicators keep them
  // mapped so the transport can change without another collective
  if (g.nproc > 1 || needs_recv_planes()) {
    for (int i = 0; i < g.nlocal; ++i) {
      cudaError_t e = cudaMalloc(&R->recv[i], 2 * R->plane);
      if (e != cudaSuccess) {
        free_registration(R.get());
        return fail(CCUBE_ERR_CUDA, "cudaMalloc(recv, %zu) failed: %s", 2 * R->plane,
                    cudaGetErrorString(e));
      }
    }
  }
  ccube_result_t rc = exchange_ptrs(R->bufs, bytes, &R->world_buf, &R->opened);
  if (rc == CCUBE_SUCCESS && R->recv[0])
    rc = exchange_ptrs(R->recv, 2 * R->plane, &R->world_recv, &R->opened);
  else
    R->world_recv.assign(g.world, nullptr);
  if (rc == CCUBE_SUCCESS) rc = build_params(R.get());
  if (rc != CCUBE_SUCCESS) {
    free_registration(R.get());
    return rc;
  }
  *out = R.get();
  g.regs.push_back(std::move(R));
  return CCUBE_SUCCESS;
}

Registration *find_registration(void *const *bufs, size_t bytes) {
  for (auto &R : g.regs) {
    if (R->bytes < bytes) continue;
    bool same = true;
    for (int i = 0; i < g.nlocal && same; ++i) same = R->bufs[i] == bufs[i];
    if (same) return R.get();
  }
  return nullptr;
}

// Block -> task placement.  Values never depend on it (every CTA is co-resident and
// a task's work is fixed by its (rank, tree, role, channel)); only which tasks share
// an SM does.  The block scheduler fills one CTA per SM before the second, so block
// b and block b + #SMs usually share an SM.
//   0: rank-major (the construction order above);
//   1: channel-major: the tasks of channel j are adjacent, so an SM pair mixes roles;
//   2: heavy first: tasks that combine children's partials (UP with children, the
//      DRAM-read-heavy stages) fill the first blocks, copies and leaves the rest, so
//      an SM rarely hosts two combining tasks.
int task_weight(const Task &x) {
  if (x.channel == kAllChannels) return 3;             // pulled leaf: no data
  if (x.role == kRoleDown || x.role == kRoleUpdate) return 2;  // copy (+ update)
  const Tree &tr = g.trees[x.tree];
  const int r = g.rank0 + x.local_rank;
  if (tr.parent[r] < 0) return 1;                      // root: 2 sources
  return tr.nchild[r] > 0 ? 0 : 2;                     // interior combine / pushed leaf
}

void order_tasks(std::vector<Task> &ts) {
  if (g.task_order == 1) {
    std::stable_sort(ts.begin(), ts.end(), [](const Task &x, const Task &y) {
      const int cx = x.channel == kAllChannels ? -1 : x.channel;
      const int cy = y.channel == kAllChannels ? -1 : y.channel;
      return cx < cy;
    });
  } else if (g.task_order == 2) {
    std::stable_sort(ts.begin(), ts.end(), [](const Task &x, const Task &y) {
      const int wx = task_weight(x), wy = task_weight(y);
      if (wx != wy) return wx < wy;
      return x.channel < y.channel;
    });
  }
}

ccube_result_t get_tasks(int channels, int overlap, TaskTable **out) {
  const bool split = split_heads_now();
  auto key = std::make_pair(channels, overlap * 2 + (g.sgd ? 1 : 0) + (split ? 4 : 0));
  auto it = g.tasks.find(key);
  if (it != g.tasks.end()) {
    *out = &it->second;
    return CCUBE_SUCCESS;
  }
  const PlanIn in = plan_in(0);
  auto task = [](int i, int t, int role, int j, int half = 0, int halves = 1, int head = 0) {
    return Task{(int16_t)i, (int16_t)t, (int16_t)role, (int16_t)j, (int16_t)half,
                (int16_t)halves, (int16_t)head};
  };
  std::vector<Task> ts, leaves;
  for (int i = 0; i < g.nlocal; ++i) {
    const int r = g.rank0 + i;
    const size_t first_leaf = leaves.size();
    for (int t = 0; t < g.ntrees; ++t) {
      const Tree &tr = g.trees[t];
      const bool root = tr.parent[r] < 0;
      if (!root && tr.nchild[r] == 0 && g.sgd)  // a leaf's fused SGD step (f2)
        for (int j = 0; j < channels; ++j) ts.push_back(task(i, t, kRoleUpdate, j));
      if (!root && tr.nchild[r] == 0 && edge_is_pull(r, tr.parent[r])) {
        leaves.push_back(task(i, t, kRoleUp, kAllChannels));
        continue;
      }
      const bool down = tr.nchild[r] > 0 && (!root || !overlap);
      const bool is_head = plan_is_head(in, tr, r);
      const bool head = split && is_head;
      for (int j = 0; j < channels; ++j) {
        ts.push_back(task(i, t, kRoleUp, j, 0, head ? 2 : 1, is_head));
        if (head) ts.push_back(task(i, t, kRoleUp, j, 1, 2, is_head));
      }
      if (down)
        for (int j = 0; j < channels; ++j) ts.push_back(task(i, t, kRoleDown, j));
    }
    // One leaf-group CTA per rank serves the trees in which the rank is a pulled leaf
    // (one tree for the single and double tree, P/2 of the rotated set's P); its
    // leaves' entries follow the grid in the table (`half` is fixed up below).
    if (leaves.size() > first_leaf)
      ts.push_back(task(i, 0, kRoleUp, kAllChannels, static_cast<int>(first_leaf),
                        static_cast<int>(leaves.size() - first_leaf)));
  }
  order_tasks(ts);
  for (Task &x : ts)
    if (x.channel == kAllChannels) x.half = static_cast<int16_t>(x.half + ts.size());
  TaskTable tt;
  tt.n = static_cast<int>(ts.size());
  ts.insert(ts.end(), leaves.begin(), leaves.end());
  CUDA_TRY(cudaMalloc(&tt.d_tasks, sizeof(Task) * ts.size()));
  CUDA_TRY(cudaMemcpy(tt.d_tasks, ts.data(), sizeof(Task) * ts.size(), cudaMemcpyHostToDevice));
  g.tasks[key] = tt;
  *out = &g.tasks[key];
  return CCUBE_SUCCESS;
}

ccube_result_t check_chunk(size_t chunk_bytes) {
  if (chunk_bytes == 0 || chunk_bytes % 16)
    return fail(CCUBE_ERR_INVALID_ARG, "chunk_bytes (%zu) must be a positive multiple of 16",
                chunk_bytes);
  if (chunk_bytes > (1ull << 31))
    return fail(CCUBE_ERR_INVALID_ARG, "chunk_bytes (%zu) too large", chunk_bytes);
  return CCUBE_SUCCESS;
}

// One-chunk calls on the LL protocol (see tree_allreduce.cu): tree 0 carries the
// chunk (a3: chunk 0 is on tree 0 for every tree kind), so the result is the chunked
// path's bit for bit; the epochs of the other trees do not move (K_t = 0).
ccube_result_t ll_impl(Registration *R, size_t count, ccube_dtype_t dtype, uint64_t E,
                       uint64_t K, void *stream) {
  const Tree &tr = g.trees[0];
  LLArgs a;
  memset(&a, 0, sizeof a);
  const uint64_t bytes = count * elem_size(dtype);
  const uint64_t lines = (bytes + 7) / 8;
  const int threads = 512;
  uint64_t ctas = (lines + 4 * threads - 1) / (4 * threads);  // <= 4 lines per thread
  if (ctas > 16) ctas = 16;
  // every LL CTA polls lines other CTAs produce: all must be co-resident (one 512-thread
  // CTA per SM is always available to this kernel's 86-register threads)
  const uint64_t per_rank_max = static_cast<uint64_t>(g.sm_count / g.nlocal);
  if (ctas > per_rank_max) ctas = per_rank_max > 0 ? per_rank_max : 1;
  a.ctas = static_cast<int>(ctas);
  a.count = count;
  a.epoch = g.ll_epoch + 1;
  a.done_base = g.ll_done;
  a.enq_value = g.base[0] + K;   // every chunk (all on tree 0) has landed
  a.err = g.err_dev;
  a.timeout_ns = g.timeout_ns;
  for (int i = 0; i < g.nlocal; ++i) {
    const int r = g.rank0 + i;
    LLRank &m = a.r[i];
    char *own = g.flags_local[i];
    m.buf = R->bufs[i];
    m.nchild = tr.nchild[r];
    for (int s = 0; s < tr.nchild[r]; ++s) {
      const int c = tr.child[r][s];
      if (!g.world_flags[c]) return fail(CCUBE_ERR_BOOTSTRAP, "child %d not mapped", c);
      m.up_in[s] = own + ll_offset(kLLUp0 + s);
      m.down_out[s] = g.world_flags[c] + ll_offset(kLLDown);
    }
    m.down_in = own + ll_offset(kLLDown);
    const int par = tr.parent[r];
    if (par >= 0) {
      if (!g.world_flags[par]) return fail(CCUBE_ERR_BOOTSTRAP, "parent %d not mapped", par);
      m.up_out = g.world_flags[par] + ll_offset(kLLUp0 + child_slot(tr, par, r));
    }
    m.enq = reinterpret_cast<uint64_t *>(own + flag_offset(0, kEnq, 0));
    m.done = reinterpret_cast<uint64_t *>(own + kLLDoneOffset);
  }
  const int rc = launch_ll(a, dtype, g.sys_scope, g.nlocal, threads, stream);
  if (rc != cudaSuccess)
    return fail(CCUBE_ERR_CUDA, "LL kernel launch failed: %s",
                cudaGetErrorString(static_cast<cudaError_t>(rc)));
  g.ll_epoch += 1;
  if (ctas > 1) g.ll_done += ctas;   // a single CTA does not count itself
  g.have_call = true;
  g.last_E = E;
  g.last_channels = 1;   // the gate waits on channel 0 of tree 0
  g.last_sgd = false;
  g.last_ctas = static_cast<int>(ctas) * g.nlocal;
  g.last_tma = 0;
  g.last_ll = 1;
  for (int t = 0; t < g.ntrees; ++t) {
    g.last_base[t] = g.base[t];
    g.last_K[t] = t == 0 ? static_cast<uint32_t>(K) : 0;
  }
  g.base[0] += K;
  return CCUBE_SUCCESS;
}

ccube_result_t allreduce_impl(void *const *bufs, size_t count, ccube_dtype_t dtype,
                              void *stream) {
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  CC_TRY(check_err_word());
  if (dtype != CCUBE_INT32 && dtype != CCUBE_FLOAT32 && dtype != CCUBE_BFLOAT16)
    return fail(CCUBE_ERR_INVALID_ARG, "bad dtype %d", (int)dtype);
  if (!bufs) return fail(CCUBE_ERR_INVALID_ARG, "bufs is NULL");
  for (int i = 0; i < g.nlocal; ++i) {
    if (!bufs[i]) return fail(CCUBE_ERR_INVALID_ARG, "buffer %d is NULL", i);
    if (reinterpret_cast<uintptr_t>(bufs[i]) % 16)
      return fail(CCUBE_ERR_INVALID_ARG, "buffer %d (%p) is not 16-byte aligned", i, bufs[i]);
  }
  const int es = elem_size(dtype);
  if (count > (~0ull) / 4) return fail(CCUBE_ERR_INVALID_ARG, "count too large");
  if (g.sgd && g.world > 1 && count > 0) {
    if (dtype != CCUBE_FLOAT32)
      return fail(CCUBE_ERR_INVALID_ARG, "the fused SGD update needs fp32 gradients");
    if (count * 4 > g.sgd_bytes)
      return fail(CCUBE_ERR_INVALID_ARG, "count %zu exceeds the registered weights (%zu bytes)",
                  count, g.sgd_bytes);
  }
  if (g.world == 1 || count == 0) return CCUBE_SUCCESS;
  const size_t bytes = count * es;
  Registration *R = find_registration(bufs, bytes);
  if (!R) CC_TRY(do_register(bufs, bytes, &R));

  const uint64_t E = g.chunk_bytes / es;
  const uint64_t K = (count + E - 1) / E;
  // one-chunk messages up to the LL threshold: the LL protocol — the same tree-0 fold,
  // one kernel without counters or fences.  (Multi-chunk single-tree messages on LL
  // measured no faster than the chunked kernel from 512 KiB up: DESIGN §10.)
  if (g.ll && !g.sgd && K == 1 && bytes <= g.ll_max)
    return ll_impl(R, count, dtype, E, K, stream);
  if (K > 0xffffffffull) return fail(CCUBE_ERR_INVALID_ARG, "too many chunks");

  // all CTAs spin on each other: they must be co-resident
  int nctl = g.split_control == 0 ? 1 : 2;  // AUTO may drop to 1 below
  // the TMA datapath needs a producer and at least one consumer data warp
  const bool tma_wanted = want_tma();
  // co-resident CTAs per GPU for a CTA of `data` data threads (occupancy, cached)
  auto capacity = [&](int data, int *cap_out, int *tma_out) -> ccube_result_t {
    const int tma_ = tma_wanted && data >= 64 ? 1 : 0;
    const int cta = data + 32 * nctl;
    auto key = std::make_pair((int)dtype * 2 + (g.sgd ? 1 : 0) + 8 * tma_, cta);
    if (!g.max_blocks.count(key)) {
      int b = 0;
      const int rc = query_max_blocks_per_sm(dtype, g.sys_scope, g.sgd, cta, tma_, &b);
      if (rc != cudaSuccess)
        return fail(CCUBE_ERR_CUDA, "occupancy query failed: %s",
                    cudaGetErrorString(static_cast<cudaError_t>(rc)));
      g.max_blocks[key] = b;
    }
    *cap_out = g.max_blocks[key] * g.sm_count;
    *tma_out = tma_;
    return CCUBE_SUCCESS;
  };
  // Launch geometry (both ends of an edge must slice chunks alike).
  // J is computed from the maximum task count over ALL processes, so it does not
  // depend on this rank's role in the trees; every setting it depends on is agreed
  // (init's Hello, the collective setters) and every GPU has the same SM count and
  // architecture (init checks it), so every rank computes the same J and the same
  // co-residency verdict without another exchange.
  const PlanIn in = plan_in(bytes);
  int data_threads = g.threads, cap = 0, tma = 0;
  if (data_threads == 0) {
    // auto CTA size: 256-thread CTAs with 6 vectors in flight per lane and source (3 KB
    // blocks) when every channel's slice of a chunk holds >= 3 units of 2 KB, so the
    // 3 KB blocks tile it; 8 data warps with 2 KB blocks when the slices are short
    // (many channels: P = 2 / 4), where fewer warps would mean fewer bytes in flight
    // (round 2).  In the 256-thread case AUTO control (CCUBE_SPLIT_CONTROL
    // unset) runs ONE control warp and 7 data warps instead of 2 + 6 once the call has
    // >= kOneControlMinChunks chunks: the data warps' registers are the bytes in
    // flight, and on a bandwidth-bound call the extra warp outweighs the poll round
    // trip a release may now wait behind (P = 8, 102 MB: single 0.3191 -> 0.3166 ms,
    // double 0.3236 -> 0.3141 ms), while a latency-bound one (<= 64 chunks: the fill
    // and drain dominate) loses 4-10% to that round trip (round 2 session
    // 2).  Deterministic in agreed quantities, like J.
    CC_TRY(capacity(kDefaultDataThreads, &cap, &tma));  // a 256-thread CTA (nctl = 2)
    const int J0 = g.channels ? g.channels : plan_auto_channels(in, cap);
    const uint64_t first = bytes < g.chunk_bytes ? bytes : g.chunk_bytes;
    const uint64_t units = (first + 2047) / 2048;
    if (units >= 3ull * J0) {
      data_threads = kDefaultDataThreads;
      if (g.split_control < 0 && !split_heads_now() && K >= kOneControlMinChunks) {
        nctl = 1;
        data_threads += 32;  // the same 256-thread CTA
      }
    } else {
      data_threads = 256;
    }
  }
  CC_TRY(capacity(data_threads, &cap, &tma));
  const int cta_threads = data_threads + 32 * nctl;  // data warps + the control warp(s)
  const int J = g.channels ? g.channels : plan_auto_channels(in, cap);
  if (plan_max_tasks(in, J) > cap)
    return fail(CCUBE_ERR_UNSUPPORTED,
                "%d CTAs (channels=%d) cannot be co-resident (capacity %d per GPU); lower "
                "channels", plan_max_tasks(in, J), J, cap);

  LaunchArgs a;
  memset(&a, 0, sizeof a);
  a.count = count;
  a.elems_per_chunk = static_cast<uint32_t>(E);
  a.ntrees = g.ntrees;
  a.nchannels = J;
  for (int t = 0; t < g.ntrees; ++t)  // chunk c travels on tree c mod T (R4)
    a.K[t] = static_cast<uint32_t>(K > static_cast<uint64_t>(t) ? (K - t + g.ntrees - 1) / g.ntrees : 0);
  for (int t = 0; t < g.ntrees; ++t) a.base[t] = g.base[t];
  a.overlap = g.overlap;
  a.timeout_ns = g.timeout_ns;
  a.err = g.err_dev;
  a.trace = g.trace;
  a.trace_kmax = static_cast<uint32_t>(g.trace_kmax);
  // profiling only (tools/pipeline_profile.py): with CCUBE_TRACE_UP=1 the trace
  // buffer is twice as long and its second half records, per (rank, tree, chunk,
  // channel), when the reduce-up partial left the rank for its parent
  if (g.trace && env_int("CCUBE_TRACE_UP", 0))
    a.trace_up = static_cast<uint64_t>(g.nlocal) * g.ntrees * g.trace_kmax * J;
  a.l2_hints = g.l2_hints;
  a.sgd = g.sgd ? 1 : 0;
  a.sgd_alpha = g.sgd_alpha;
  a.tma = tma;
  a.split_control = nctl == 2 ? 1 : 0;
  a.backoff_ns = g.backoff_ns;
  a.debug_nodep = g.debug_nodep;
  a.elem_size = static_cast<int>(es);
  a.params = R->d_params;

  TaskTable *tt = nullptr;
  CC_TRY(get_tasks(J, g.overlap, &tt));
  a.tasks = tt->d_tasks;

  const int rc = launch_tree_allreduce(a, dtype, g.sys_scope, tt->n, cta_threads, stream);
  if (rc != cudaSuccess)
    return fail(CCUBE_ERR_CUDA, "kernel launch failed: %s",
                cudaGetErrorString(static_cast<cudaError_t>(rc)));
  g.have_call = true;
  g.last_E = E;
  g.last_channels = J;
  g.last_sgd = g.sgd;
  g.last_ctas = tt->n;
  g.last_tma = tma;
  g.last_threads = data_threads;
  g.last_ll = 0;
  for (int t = 0; t < g.ntrees; ++t) {
    g.last_base[t] = g.base[t];
    g.last_K[t] = a.K[t];
    g.base[t] += a.K[t];
  }
  return CCUBE_SUCCESS;
}

ccube_result_t gradq_wait_impl(int local_rank, int layer_id, void *stream) {
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  CC_TRY(check_err_word());
  if (local_rank < 0 || local_rank >= g.nlocal)
    return fail(CCUBE_ERR_INVALID_ARG, "local_rank %d out of range", local_rank);
  if (layer_id < 0 || layer_id >= static_cast<int>(g.layer_ends.size()))
    return fail(CCUBE_ERR_INVALID_ARG, "layer_id %d out of range (%zu layers set)", layer_id,
                g.layer_ends.size());
  if (g.world == 1 || !g.have_call) return CCUBE_SUCCESS;
  // LCT[l] = ceil(end_l / E) chunks (R9, R10); tree t needs its share (R4)
  uint64_t total_K = 0;
  for (int t = 0; t < g.ntrees; ++t) total_K += g.last_K[t];
  uint64_t lct = (g.layer_ends[layer_id] + g.last_E - 1) / g.last_E;
  if (lct > total_K) lct = total_K;
  // tree t carries chunks t, t+T, ...: layer l needs ceil((LCT - t) / T) of them
  uint64_t need[kMaxTrees] = {};
  for (int t = 0; t < g.ntrees; ++t)
    need[t] = lct > static_cast<uint64_t>(t) ? (lct - t + g.ntrees - 1) / g.ntrees : 0;
  std::vector<const uint64_t *> ctr;
  std::vector<uint64_t> tgt;
  for (int t = 0; t < g.ntrees; ++t) {
    if (need[t] == 0) continue;
    for (int j = 0; j < g.last_channels; ++j) {
      // with the fused update the gate opens once the WEIGHTS of the chunk are updated
      ctr.push_back(reinterpret_cast<const uint64_t *>(
          g.flags_local[local_rank] + flag_offset(t, g.last_sgd ? kUpd : kEnq, j)));
      tgt.push_back(g.last_base[t] + need[t]);
    }
  }
  // waits are idempotent ">=" checks, so they may be split into batches freely
  size_t done = 0;
  if (g.use_memop) {
    load_driver();
    while (g_drv.batchMemOp && done < ctr.size()) {
      const size_t n = std::min(ctr.size() - done, static_cast<size_t>(kMaxGateCounters));
      std::vector<CUstreamBatchMemOpParams> ops(n);
      for (size_t i = 0; i < n; ++i) {
        memset(&ops[i], 0, sizeof ops[i]);
        ops[i].waitValue.operation = CU_STREAM_MEM_OP_WAIT_VALUE_64;
        ops[i].waitValue.address = reinterpret_cast<CUdeviceptr>(ctr[done + i]);
        ops[i].waitValue.value64 = tgt[done + i];
        ops[i].waitValue.flags =
            CU_STREAM_WAIT_VALUE_GEQ | (g.gate_flush ? CU_STREAM_WAIT_VALUE_FLUSH : 0);
      }
      if (g_drv.batchMemOp(static_cast<CUstream>(stream), static_cast<unsigned>(n), ops.data(),
                           0) != CUDA_SUCCESS)
        break;
      done += n;
    }
    if (done == ctr.size()) return CCUBE_SUCCESS;
    g.use_memop = false;  // fall back to the spin-gate kernel from now on
  }
  while (done < ctr.size()) {
    const int n = static_cast<int>(std::min(ctr.size() - done, static_cast<size_t>(kMaxGateCounters)));
    const int rc = launch_gate(ctr.data() + done, tgt.data() + done, n, g.err_dev, g.timeout_ns,
                               g.sys_scope, stream);
    if (rc != cudaSuccess)
      return fail(CCUBE_ERR_CUDA, "gate launch failed: %s",
                  cudaGetErrorString(static_cast<cudaError_t>(rc)));
    done += n;
  }
  return CCUBE_SUCCESS;
}

void release_all() {
  for (auto &R : g.regs) free_registration(R.get());
  g.regs.clear();
  for (void *b : g.opened_flags) ipc_close(b);
  g.opened_flags.clear();
  for (char *f : g.flags_local)
    if (f) cudaFree(f);
  g.flags_local.clear();
  g.world_flags.clear();
  for (auto &kv : g.tasks) cudaFree(kv.second.d_tasks);
  g.tasks.clear();
  if (g.err_host) cudaFreeHost(g.err_host);
  g.err_host = g.err_dev = nullptr;
  g.max_blocks.clear();
}

struct Hello {
  uint32_t magic;
  int32_t world, nlocal, rank, tree_kind, device;
  // settings that fix which bytes a counter covers or how a chunk is sliced: every
  // rank must start from the same ones (CCUBE_* environment)
  int32_t channels, threads, datapath, transport, l2_hints, split_control;
  // the launch geometry is computed locally from the occupancy: every GPU must be
  // the same architecture with the same SM count
  int32_t sm_count, cc_major, cc_minor, ll;
  uint64_t ll_max;
  int32_t split_heads, pad2;
  uint64_t chunk_bytes;
  char busid[32];
  int8_t place[CCUBE_MAX_RANKS];  // the placement (R19), identity when none was set
};

// Placement set by ccube_set_placement for the next ccube_init (0 = identity).  Lives
// outside Comm: it is configuration, kept across finalize/init.
int g_place[CCUBE_MAX_RANKS];
int g_place_P = 0;

bool is_permutation(const int *perm, int P) {
  bool seen[CCUBE_MAX_RANKS] = {};
  for (int v = 0; v < P; ++v) {
    if (perm[v] < 0 || perm[v] >= P || seen[perm[v]]) return false;
    seen[perm[v]] = true;
  }
  return true;
}

ccube_result_t barrier_impl(void *stream) {
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  CC_TRY(check_err_word());
  if (g.nproc == 1) return CCUBE_SUCCESS;  // one process: stream order is the barrier
  const Tree &tr = g.trees[0];
  std::vector<BarrierRank> br(g.nlocal);
  for (int i = 0; i < g.nlocal; ++i) {
    const int r = g.rank0 + i;
    BarrierRank &b = br[i];
    memset(&b, 0, sizeof b);
    char *own = g.flags_local[i];
    b.nchild = tr.nchild[r];
    for (int s = 0; s < tr.nchild[r]; ++s) {
      const int c = tr.child[r][s];
      if (!g.world_flags[c]) return fail(CCUBE_ERR_BOOTSTRAP, "child %d not mapped", c);
      b.arrive[s] = reinterpret_cast<const uint64_t *>(own + barrier_offset(kBarArrive0 + s));
      b.child_release[s] = reinterpret_cast<uint64_t *>(g.world_flags[c] + barrier_offset(kBarRelease));
    }
    b.release = reinterpret_cast<const uint64_t *>(own + barrier_offset(kBarRelease));
    const int par = tr.parent[r];
    if (par >= 0) {
      if (!g.world_flags[par]) return fail(CCUBE_ERR_BOOTSTRAP, "parent %d not mapped", par);
      b.parent_arrive = reinterpret_cast<uint64_t *>(
          g.world_flags[par] + barrier_offset(kBarArrive0 + child_slot(tr, par, r)));
    }
  }
  const int rc = launch_barrier(br.data(), g.nlocal, g.bar_epoch + 1, g.err_dev, g.timeout_ns,
                                g.sys_scope, stream);
  if (rc != cudaSuccess)
    return fail(CCUBE_ERR_CUDA, "barrier launch failed: %s",
                cudaGetErrorString(static_cast<cudaError_t>(rc)));
  ++g.bar_epoch;
  return CCUBE_SUCCESS;
}


// ccube_measure_peer_bandwidth (SURVEY §8(d) "P2P port-peak microbenchmark"): the
// AllReduce's own cross-GPU data path — 128-bit loads from local HBM, 128-bit
// stores into a peer's HBM over NVLink / NVSwitch — timed on the device after a
// device-side barrier, one destination per GPU at a time (every rank shifted by
// the same k, so every port carries one stream each way) and fanned out to m peers.
ccube_result_t peer_bandwidth_impl(size_t bytes, int iters, double *pair_gbs, double *fanout_gbs) {
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  CC_TRY(check_err_word());
  if (g.nlocal != 1 || g.nproc < 2)
    return fail(CCUBE_ERR_UNSUPPORTED, "peer bandwidth needs one process per GPU (nlocal == 1)");
  if (bytes == 0 || bytes % 16 || iters < 1 || !pair_gbs || !fanout_gbs)
    return fail(CCUBE_ERR_INVALID_ARG, "bytes must be a positive multiple of 16, iters >= 1");
  const int P = g.world, me = g.rank0;
  char *src = nullptr, *recv = nullptr;
  std::vector<char *> world_recv;
  std::vector<void *> opened;
  cudaStream_t st = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  std::vector<double> mine(2 * P, 0.0);
  ccube_result_t rc = CCUBE_SUCCESS;
  auto cuda_ok = [&](cudaError_t e, const char *what) {
    if (e != cudaSuccess && rc == CCUBE_SUCCESS)
      rc = fail(CCUBE_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
    return rc == CCUBE_SUCCESS;
  };
  if (cuda_ok(cudaMalloc(&src, bytes), "cudaMalloc(src)") &&
      cuda_ok(cudaMalloc(&recv, bytes * P), "cudaMalloc(recv)") &&
      cuda_ok(cudaMemset(src, 0x5a, bytes), "cudaMemset") &&
      cuda_ok(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking), "stream") &&
      cuda_ok(cudaEventCreate(&e0), "event") && cuda_ok(cudaEventCreate(&e1), "event") &&
      cuda_ok(cudaDeviceSynchronize(), "sync"))
    rc = exchange_ptrs(std::vector<char *>{recv}, bytes * P, &world_recv, &opened, true);
  const int grid = 2 * g.sm_count;
  auto timed = [&](const std::vector<char *> &dst) -> double {
    double best = 1e30;
    for (int it = 0; it < iters && rc == CCUBE_SUCCESS; ++it) {
      rc = barrier_impl(st);
      if (rc != CCUBE_SUCCESS) break;
      cuda_ok(cudaEventRecord(e0, st), "record");
      const int lr = launch_peer_copy(src, dst.data(), static_cast<int>(dst.size()), bytes, grid, st);
      cuda_ok(static_cast<cudaError_t>(lr), "peer copy launch");
      cuda_ok(cudaEventRecord(e1, st), "record");
      if (!cuda_ok(cudaEventSynchronize(e1), "sync")) break;
      rc = check_err_word();
      if (rc != CCUBE_SUCCESS) break;
      float ms = 0;
      cuda_ok(cudaEventElapsedTime(&ms, e0, e1), "elapsed");
      best = std::min(best, static_cast<double>(ms) * 1e-3);
    }
    return best;
  };
  for (int k = 1; k < P && rc == CCUBE_SUCCESS; ++k) {  // pairs: every rank shifted by k
    const int d = (me + k) % P;
    const double t = timed({world_recv[d] + static_cast<size_t>(me) * bytes});
    mine[d] = bytes / t / 1e9;
  }
  for (int m = 1; m < P && rc == CCUBE_SUCCESS; ++m) {  // fan-out to m peers at once
    std::vector<char *> dst;
    for (int q = 1; q <= m; ++q)
      dst.push_back(world_recv[(me + q) % P] + static_cast<size_t>(me) * bytes);
    const double t = timed(dst);
    mine[P + m] = static_cast<double>(m) * bytes / t / 1e9;
  }
  // every rank reaches this exchange (a failed rank sends NaNs), then peers stop
  // using our memory before anything is unmapped or freed
  if (rc != CCUBE_SUCCESS) std::fill(mine.begin(), mine.end(), -1.0);
  std::vector<double> all(2 * P * g.nproc);
  const ccube_result_t grc = do_allgather(mine.data(), all.data(), sizeof(double) * 2 * P);
  if (rc == CCUBE_SUCCESS) rc = grc;
  for (int p = 0; p < g.nproc && rc == CCUBE_SUCCESS; ++p)
    if (all[2 * P * p] < 0) rc = fail(CCUBE_ERR_CUDA, "peer bandwidth failed on process %d", p);
  if (rc == CCUBE_SUCCESS) {
    for (int i = 0; i < P; ++i)
      for (int j = 0; j < P; ++j) pair_gbs[i * P + j] = all[2 * P * i + j];
    fanout_gbs[0] = 0.0;
    for (int m = 1; m < P; ++m) {
      double lo = 1e30;
      for (int i = 0; i < P; ++i) lo = std::min(lo, all[2 * P * i + P + m]);
      fanout_gbs[m] = lo;
    }
  }
  for (void *b : opened) ipc_close(b);
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (st) cudaStreamDestroy(st);
  if (src) cudaFree(src);
  if (recv) cudaFree(recv);
  return rc;
}

}  // namespace
}  // namespace ccube

using namespace ccube;

extern "C" {

ccube_result_t ccube_init(const ccube_world_t *world, ccube_tree_kind_t tree_kind,
                          size_t chunk_bytes) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g.init) return fail(CCUBE_ERR_ALREADY_INITIALIZED, "already initialized");
  if (!world) return fail(CCUBE_ERR_INVALID_ARG, "world is NULL");
  const int P = world->world_size;
  if (P < 1) return fail(CCUBE_ERR_INVALID_ARG, "world_size %d < 1", P);
  if (P > CCUBE_MAX_RANKS)
    return fail(CCUBE_ERR_UNSUPPORTED, "world_size %d > %d (one NVSwitch domain)", P,
                CCUBE_MAX_RANKS);
  if (world->nlocal < 1 || P % world->nlocal)
    return fail(CCUBE_ERR_INVALID_ARG, "nlocal %d must divide world_size %d", world->nlocal, P);
  if (world->rank < 0 || world->rank >= P || world->rank % world->nlocal)
    return fail(CCUBE_ERR_INVALID_ARG, "rank %d must be a multiple of nlocal in [0, %d)",
                world->rank, P);
  if (tree_kind != CCUBE_TREE_SINGLE && tree_kind != CCUBE_TREE_DOUBLE &&
      tree_kind != CCUBE_TREE_ROTATED)
    return fail(CCUBE_ERR_INVALID_ARG, "bad tree kind %d", (int)tree_kind);
  if (world->nlocal < P && !world->allgather)
    return fail(CCUBE_ERR_INVALID_ARG, "allgather callback required when nlocal < world_size");
  if (g_place_P != 0 && g_place_P != P)
    return fail(CCUBE_ERR_INVALID_ARG, "the placement was set for %d ranks, world_size is %d",
                g_place_P, P);
  if (chunk_bytes == 0) chunk_bytes = CCUBE_DEFAULT_CHUNK_BYTES;
  int channels = env_int("CCUBE_CHANNELS", 0);
  if (channels < 0 || channels > CCUBE_MAX_CHANNELS)
    return fail(CCUBE_ERR_INVALID_ARG, "CCUBE_CHANNELS %d out of range", channels);
  CC_TRY(check_chunk(chunk_bytes));
  int threads = env_int("CCUBE_THREADS", 0);
  if (threads != 0 && (threads < 32 || threads > 256 || threads % 32))
    return fail(CCUBE_ERR_INVALID_ARG, "CCUBE_THREADS %d out of range [32, 256] (0 = auto)",
                threads);
  const int transport = env_int("CCUBE_TRANSPORT", CCUBE_TRANSPORT_AUTO);
  if (transport < CCUBE_TRANSPORT_AUTO || transport > CCUBE_TRANSPORT_PULL)
    return fail(CCUBE_ERR_INVALID_ARG, "CCUBE_TRANSPORT %d out of range", transport);

  g = Comm();
  g.world = P;
  g.rank0 = world->rank;
  g.nlocal = world->nlocal;
  g.device = world->cuda_device;
  g.nproc = P / world->nlocal;
  g.proc = world->rank / world->nlocal;
  g.allgather = world->allgather;
  g.ctx = world->ctx;
  g.tree_kind = tree_kind;
  g.ntrees = num_trees(P, tree_kind);
  g.chunk_bytes = chunk_bytes;
  g.channels = channels;
  g.threads = threads;
  g.transport = transport;
  g.overlap = 1;
  g.l2_hints = env_int("CCUBE_L2_HINTS", 1);
  {
    const int sc = env_int("CCUBE_SPLIT_CONTROL", -1);
    g.split_control = sc < 0 ? -1 : (sc != 0 ? 1 : 0);
  }
  g.task_order = env_int("CCUBE_TASK_ORDER", 0);
  g.backoff_ns = env_int("CCUBE_BACKOFF_NS", 64);
  g.debug_nodep = env_int("CCUBE_DEBUG_NODEP", 0);
  g.ll = env_int("CCUBE_LL", 1) != 0 ? 1 : 0;
  // off by default: measured slower (round 2) — the head then outruns the
  // stages after it, which lose CTAs and the L2 residency of the head's partials
  g.split_heads = env_int("CCUBE_SPLIT_HEADS", 0) != 0 ? 1 : 0;
  {
    const int m = env_int("CCUBE_LL_MAX_BYTES", static_cast<int>(kLLDefaultMaxBytes));
    g.ll_max = m < 0 ? 0 : (static_cast<uint64_t>(m) > kLLMaxBytes ? kLLMaxBytes : m);
  }
  g.datapath = env_int("CCUBE_DATAPATH", CCUBE_DATAPATH_AUTO);
  if (g.datapath != CCUBE_DATAPATH_LSU && g.datapath != CCUBE_DATAPATH_TMA)
    g.datapath = CCUBE_DATAPATH_AUTO;
  g.sys_scope = g.nproc > 1;
  g.timeout_ns = static_cast<uint64_t>(env_int("CCUBE_WATCHDOG_MS", 10000)) * 1000000ull;
  g.use_memop = env_int("CCUBE_GATE_KERNEL", 0) == 0;
  for (int t = 0; t < g.ntrees; ++t) {
    build_tree(P, tree_kind, t, &g.trees[t]);
    if (g_place_P == P) place_tree(g_place, &g.trees[t]);
  }

  // (i) config agreement — host only, so it also runs (and can be tested) without a GPU
  Hello mine;
  memset(&mine, 0, sizeof mine);
  mine.magic = 0xCC0BE001u;
  mine.world = P;
  mine.nlocal = g.nlocal;
  mine.rank = g.rank0;
  mine.tree_kind = tree_kind;
  mine.device = g.device;
  mine.chunk_bytes = chunk_bytes;
  mine.channels = g.channels;
  mine.threads = g.threads;
  mine.datapath = g.datapath;
  mine.transport = g.transport;
  mine.l2_hints = g.l2_hints;
  mine.split_control = g.split_control;
  mine.ll = g.ll;
  mine.ll_max = g.ll_max;
  mine.split_heads = g.split_heads;
  if (cudaDeviceGetAttribute(&mine.sm_count, cudaDevAttrMultiProcessorCount, g.device) !=
          cudaSuccess ||
      cudaDeviceGetAttribute(&mine.cc_major, cudaDevAttrComputeCapabilityMajor, g.device) !=
          cudaSuccess ||
      cudaDeviceGetAttribute(&mine.cc_minor, cudaDevAttrComputeCapabilityMinor, g.device) !=
          cudaSuccess) {
    cudaGetLastError();
    mine.sm_count = mine.cc_major = mine.cc_minor = -1;  // no GPU: CUDA setup fails below
  }
  for (int v = 0; v < P; ++v) mine.place[v] = static_cast<int8_t>(g_place_P == P ? g_place[v] : v);
  if (cudaDeviceGetPCIBusId(mine.busid, sizeof mine.busid, g.device) != cudaSuccess)
    snprintf(mine.busid, sizeof mine.busid, "nodevice-%d", g.rank0);
  std::vector<Hello> all(g.nproc);
  ccube_result_t rc = do_allgather(&mine, all.data(), sizeof(Hello));
  if (rc != CCUBE_SUCCESS) {
    g = Comm();
    return rc;
  }
  const bool allow_shared = env_int("CCUBE_ALLOW_SHARED_GPU", 0) != 0;
  for (int p = 0; p < g.nproc; ++p) {
    const Hello &h = all[p];
    if (h.magic != mine.magic || h.world != P || h.nlocal != g.nlocal ||
        h.rank != p * g.nlocal || h.tree_kind != mine.tree_kind ||
        h.chunk_bytes != mine.chunk_bytes || memcmp(h.place, mine.place, sizeof h.place)) {
      g = Comm();
      return fail(CCUBE_ERR_INVALID_ARG,
                  "ranks disagree on the configuration (process %d: world %d nlocal %d rank %d "
                  "tree %d chunk %llu, or the placement)",
                  p, h.world, h.nlocal, h.rank, h.tree_kind, (unsigned long long)h.chunk_bytes);
    }
    if (h.sm_count != mine.sm_count || h.cc_major != mine.cc_major ||
        h.cc_minor != mine.cc_minor) {
      g = Comm();
      return fail(CCUBE_ERR_UNSUPPORTED,
                  "mixed GPUs (process %d: sm_%d%d with %d SMs; here sm_%d%d with %d SMs): "
                  "the launch geometry needs identical GPUs",
                  p, h.cc_major, h.cc_minor, h.sm_count, mine.cc_major, mine.cc_minor,
                  mine.sm_count);
    }
    if (h.channels != mine.channels || h.threads != mine.threads ||
        h.datapath != mine.datapath || h.transport != mine.transport ||
        h.l2_hints != mine.l2_hints || h.split_control != mine.split_control ||
        h.ll != mine.ll || h.ll_max != mine.ll_max || h.split_heads != mine.split_heads) {
      g = Comm();
      return fail(CCUBE_ERR_INVALID_ARG,
                  "ranks disagree on the launch settings (process %d: CCUBE_CHANNELS %d "
                  "CCUBE_THREADS %d CCUBE_DATAPATH %d CCUBE_TRANSPORT %d CCUBE_L2_HINTS %d "
                  "CCUBE_SPLIT_CONTROL %d, or CCUBE_LL[_MAX_BYTES] / CCUBE_SPLIT_HEADS; here "
                  "%d %d %d %d %d %d)",
                  p, h.channels, h.threads, h.datapath, h.transport, h.l2_hints,
                  h.split_control, mine.channels, mine.threads, mine.datapath, mine.transport,
                  mine.l2_hints, mine.split_control);
    }
    // Several processes on one GPU only time-slice (no MPS): their spinning kernels
    // make progress one context switch at a time.  Refused unless a test asks for it
    // (CCUBE_ALLOW_SHARED_GPU=1 exercises the IPC / .sys-scope path on one GPU).
    for (int q = 0; q < p && !allow_shared; ++q)
      if (strncmp(all[q].busid, h.busid, sizeof h.busid) == 0 &&
          strncmp(h.busid, "nodevice", 8) != 0) {
        g = Comm();
        return fail(CCUBE_ERR_UNSUPPORTED,
                    "processes %d and %d share GPU %s: the spinning kernels of two processes "
                    "only time-slice on one GPU (CCUBE_ALLOW_SHARED_GPU=1 permits it for tests)",
                    q, p, h.busid);
      }
  }

  // (ii) CUDA setup
  cudaError_t ce = cudaSetDevice(g.device);
  if (ce != cudaSuccess) {
    g = Comm();
    return fail(CCUBE_ERR_CUDA, "cudaSetDevice(%d): %s", world->cuda_device,
                cudaGetErrorString(ce));
  }
  auto bail = [&](ccube_result_t r) {
    release_all();
    g = Comm();
    return r;
  };
  int major = 0;
  if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, g.device) != cudaSuccess ||
      cudaDeviceGetAttribute(&g.sm_count, cudaDevAttrMultiProcessorCount, g.device) != cudaSuccess)
    return bail(fail(CCUBE_ERR_CUDA, "device attribute query failed"));
  if (major != 10)
    return bail(fail(CCUBE_ERR_UNSUPPORTED, "compute capability %d.x: built for sm_100a only",
                     major));
  ce = cudaHostAlloc(reinterpret_cast<void **>(&g.err_host), 4 * sizeof(int), cudaHostAllocMapped);
  if (ce != cudaSuccess) return bail(fail(CCUBE_ERR_CUDA, "cudaHostAlloc: %s", cudaGetErrorString(ce)));
  memset(g.err_host, 0, 4 * sizeof(int));
  ce = cudaHostGetDevicePointer(reinterpret_cast<void **>(&g.err_dev), g.err_host, 0);
  if (ce != cudaSuccess) return bail(fail(CCUBE_ERR_CUDA, "cudaHostGetDevicePointer: %s", cudaGetErrorString(ce)));
  // (iii) peer access (SURVEY §8(b) validation): every tree neighbour on another GPU
  // must be reachable with device loads/stores (NVLink / NVSwitch).  Decided
  // collectively, so every rank either proceeds or returns UNSUPPORTED.
  if (g.nproc > 1) {
    int32_t ok = 1;
    char why[200] = "";
    for (int r = 0; r < g.world && ok; ++r) {
      if (is_local(r) || !is_neighbor_of_local(r)) continue;
      const Hello &h = all[r / g.nlocal];
      if (strncmp(h.busid, mine.busid, sizeof h.busid) == 0) continue;  // shared GPU (tests)
      int dev = -1;
      if (cudaDeviceGetByPCIBusId(&dev, h.busid) != cudaSuccess) {
        cudaGetLastError();  // the peer's GPU is not visible here: the IPC open decides
        continue;
      }
      int can = 0;
      if (cudaDeviceCanAccessPeer(&can, g.device, dev) != cudaSuccess) can = 0;
      if (!can) {
        ok = 0;
        snprintf(why, sizeof why, "GPU %s (rank %d) cannot access GPU %s (rank %d) as a peer",
                 mine.busid, g.rank0, h.busid, r);
      }
    }
    std::vector<int32_t> oks(g.nproc);
    rc = do_allgather(&ok, oks.data(), sizeof ok);
    if (rc != CCUBE_SUCCESS) return bail(rc);
    for (int p = 0; p < g.nproc; ++p)
      if (!oks[p])
        return bail(fail(CCUBE_ERR_UNSUPPORTED, "no peer access between tree neighbours (%s)",
                         ok ? "reported by another process" : why));
    // gate (a9) across GPUs: the data and the Enqueue Semaphore arrive as remote
    // writes.  A stream memory-op wait is not an acquire in the PTX memory model;
    // CU_STREAM_WAIT_VALUE_FLUSH makes earlier remote writes visible to the work
    // that follows.  Without it the gate is the ld.acquire.sys spin kernel.
    int flush = 0;
    if (cudaDeviceGetAttribute(&flush, cudaDevAttrCanFlushRemoteWrites, g.device) != cudaSuccess)
      flush = 0;
    g.gate_flush = flush != 0;
    if (!g.gate_flush) g.use_memop = false;
  }
  g.flags_local.assign(g.nlocal, nullptr);
  for (int i = 0; i < g.nlocal; ++i) {
    ce = cudaMalloc(&g.flags_local[i], kWorkspaceBytes);
    if (ce == cudaSuccess) ce = cudaMemset(g.flags_local[i], 0, kWorkspaceBytes);
    if (ce != cudaSuccess) return bail(fail(CCUBE_ERR_CUDA, "flag workspace: %s", cudaGetErrorString(ce)));
  }
  ce = cudaDeviceSynchronize();
  if (ce != cudaSuccess) return bail(fail(CCUBE_ERR_CUDA, "sync: %s", cudaGetErrorString(ce)));
  g.init = true;  // exchange_ptrs needs the topology fields
  rc = exchange_ptrs(g.flags_local, kWorkspaceBytes, &g.world_flags, &g.opened_flags);
  if (rc != CCUBE_SUCCESS) return bail(rc);
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_register_buffers(void *const *bufs, size_t bytes) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  if (g.world == 1) return CCUBE_SUCCESS;
  if (bufs && find_registration(bufs, bytes)) return CCUBE_SUCCESS;
  Registration *R = nullptr;
  return do_register(bufs, bytes, &R);
}

ccube_result_t ccube_deregister_buffers(void *const *bufs) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  if (!bufs) return fail(CCUBE_ERR_INVALID_ARG, "bufs is NULL");
  if (g.world == 1) return CCUBE_SUCCESS;
  for (size_t k = 0; k < g.regs.size(); ++k) {
    bool same = true;
    for (int i = 0; i < g.nlocal && same; ++i) same = g.regs[k]->bufs[i] == bufs[i];
    if (!same) continue;
    CUDA_TRY(cudaDeviceSynchronize());
    if (g.nproc > 1) {  // peers must stop using our memory before we unmap theirs
      std::vector<int> dummy(g.nproc);
      int one = 1;
      CC_TRY(do_allgather(&one, dummy.data(), sizeof(int)));
    }
    free_registration(g.regs[k].get());
    g.regs.erase(g.regs.begin() + k);
    return CCUBE_SUCCESS;
  }
  return fail(CCUBE_ERR_INVALID_ARG, "buffer not registered");
}

ccube_result_t ccube_allreduce_tree(void *buf, size_t count, ccube_dtype_t dtype, void *stream) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g.init && g.nlocal != 1)
    return fail(CCUBE_ERR_INVALID_ARG,
                "this process hosts %d ranks: use ccube_allreduce_tree_local", g.nlocal);
  void *bufs[1] = {buf};
  return allreduce_impl(bufs, count, dtype, stream);
}

ccube_result_t ccube_allreduce_tree_local(void *const *bufs, size_t count, ccube_dtype_t dtype,
                                          void *stream) {
  std::lock_guard<std::mutex> lk(g_mu);
  return allreduce_impl(bufs, count, dtype, stream);
}

ccube_result_t ccube_barrier(void *stream) {
  std::lock_guard<std::mutex> lk(g_mu);
  return barrier_impl(stream);
}

ccube_result_t ccube_measure_peer_bandwidth(size_t bytes, int iters, double *pair_gbs,
                                            double *fanout_gbs) {
  std::lock_guard<std::mutex> lk(g_mu);
  return peer_bandwidth_impl(bytes, iters, pair_gbs, fanout_gbs);
}

ccube_result_t ccube_plan_launch(int P, ccube_tree_kind_t kind, int nlocal, int rank,
                                 size_t bytes, size_t chunk_bytes, int overlap, int channels,
                                 int cap_ctas, int *channels_out, int *ctas_out,
                                 int *max_ctas_out) {
  if (P < 1 || P > CCUBE_MAX_RANKS || nlocal < 1 || P % nlocal || rank < 0 || rank >= P)
    return fail(CCUBE_ERR_INVALID_ARG, "bad P %d, nlocal %d or rank %d", P, nlocal, rank);
  if (kind != CCUBE_TREE_SINGLE && kind != CCUBE_TREE_DOUBLE && kind != CCUBE_TREE_ROTATED)
    return fail(CCUBE_ERR_INVALID_ARG, "bad tree kind %d", (int)kind);
  if ((overlap != 0 && overlap != 1) || channels < 0 || channels > CCUBE_MAX_CHANNELS ||
      cap_ctas < 1 || !channels_out || !ctas_out || !max_ctas_out)
    return fail(CCUBE_ERR_INVALID_ARG, "bad overlap, channels, cap or output pointer");
  if (chunk_bytes == 0) chunk_bytes = CCUBE_DEFAULT_CHUNK_BYTES;
  CC_TRY(check_chunk(chunk_bytes));
  Tree trees[kMaxTrees];
  const int T = num_trees(P, kind);
  for (int t = 0; t < T; ++t) build_tree(P, kind, t, &trees[t]);
  PlanIn in;
  in.trees = trees;
  in.ntrees = T;
  in.world = P;
  in.nlocal = nlocal;
  in.transport = CCUBE_TRANSPORT_AUTO;
  in.overlap = overlap;
  in.sgd = false;
  in.bytes = bytes;
  in.chunk_bytes = chunk_bytes;
  in.split_heads = false;   // the default (CCUBE_SPLIT_HEADS=0)
  const int J = channels ? channels : plan_auto_channels(in, cap_ctas);
  *channels_out = J;
  *ctas_out = plan_tasks_of_proc(in, rank / nlocal, J);
  *max_ctas_out = plan_max_tasks(in, J);
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_gradq_set_layers(const size_t *layer_end_elems, int n_layers) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  if (n_layers < 0 || (n_layers > 0 && !layer_end_elems))
    return fail(CCUBE_ERR_INVALID_ARG, "bad layer table");
  for (int l = 1; l < n_layers; ++l)
    if (layer_end_elems[l] < layer_end_elems[l - 1])
      return fail(CCUBE_ERR_INVALID_ARG, "layer_end_elems must be nondecreasing (layer %d)", l);
  g.layer_ends.assign(layer_end_elems, layer_end_elems + n_layers);
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_gradq_wait(int layer_id, void *stream) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g.init && g.nlocal != 1)
    return fail(CCUBE_ERR_INVALID_ARG, "this process hosts %d ranks: use ccube_gradq_wait_local",
                g.nlocal);
  return gradq_wait_impl(0, layer_id, stream);
}

ccube_result_t ccube_gradq_wait_local(int local_rank, int layer_id, void *stream) {
  std::lock_guard<std::mutex> lk(g_mu);
  return gradq_wait_impl(local_rank, layer_id, stream);
}

ccube_result_t ccube_set_overlap(int on) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  const ccube_result_t v = on != 0 && on != 1
                               ? fail(CCUBE_ERR_INVALID_ARG, "overlap must be 0 or 1")
                               : CCUBE_SUCCESS;
  CC_TRY(agree_setting("overlap", on, v));
  g.overlap = on;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_gradq_set_sgd(void *const *weights, size_t bytes, float alpha) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  ccube_result_t v = CCUBE_SUCCESS;
  if (weights) {
    if (g.world < 2)
      v = fail(CCUBE_ERR_UNSUPPORTED, "the fused SGD update rides on the AllReduce (P >= 2)");
    else if (bytes == 0 || bytes % 4)
      v = fail(CCUBE_ERR_INVALID_ARG, "bad weight bytes %zu", bytes);
    for (int i = 0; i < g.nlocal && v == CCUBE_SUCCESS; ++i) {
      if (!weights[i])
        v = fail(CCUBE_ERR_INVALID_ARG, "weights[%d] is NULL", i);
      else if (reinterpret_cast<uintptr_t>(weights[i]) % 16)
        v = fail(CCUBE_ERR_INVALID_ARG, "weights[%d] is not 16-byte aligned", i);
    }
  }
  CC_TRY(agree_setting("the fused SGD update (on/off)", weights ? 1 : 0, v));
  if (!weights) {
    g.sgd = false;
    g.sgd_w.clear();
    g.sgd_bytes = 0;
  } else {
    g.sgd = true;
    g.sgd_alpha = alpha;
    g.sgd_bytes = bytes;
    g.sgd_w.assign(g.nlocal, nullptr);
    for (int i = 0; i < g.nlocal; ++i) g.sgd_w[i] = static_cast<char *>(weights[i]);
  }
  for (auto &R : g.regs) CC_TRY(build_params(R.get()));  // weights are per-rank params
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_set_channels(int channels) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  const ccube_result_t v =
      channels < 0 || channels > CCUBE_MAX_CHANNELS
          ? fail(CCUBE_ERR_INVALID_ARG, "channels %d out of range [0 (auto), %d]", channels,
                 CCUBE_MAX_CHANNELS)
          : CCUBE_SUCCESS;
  CC_TRY(agree_setting("channels", channels, v));
  g.channels = channels;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_set_threads(int threads) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  const ccube_result_t v =
      threads != 0 && (threads < 32 || threads > 256 || threads % 32)
          ? fail(CCUBE_ERR_INVALID_ARG,
                 "threads %d out of range [32, 256] (multiple of 32; 0 = auto)", threads)
          : CCUBE_SUCCESS;
  CC_TRY(agree_setting("threads", threads, v));
  g.threads = threads;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_set_datapath(int datapath) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  const ccube_result_t v = datapath != CCUBE_DATAPATH_LSU && datapath != CCUBE_DATAPATH_TMA &&
                                   datapath != CCUBE_DATAPATH_AUTO
                               ? fail(CCUBE_ERR_INVALID_ARG, "datapath %d out of range", datapath)
                               : CCUBE_SUCCESS;
  CC_TRY(agree_setting("datapath", datapath, v));
  g.datapath = datapath;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_set_protocol(int ll) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  const ccube_result_t v = ll != 0 && ll != 1
                               ? fail(CCUBE_ERR_INVALID_ARG, "protocol must be 0 or 1")
                               : CCUBE_SUCCESS;
  CC_TRY(agree_setting("the LL protocol (on/off)", ll, v));
  g.ll = ll;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_set_transport(int mode) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  const ccube_result_t v = mode < CCUBE_TRANSPORT_AUTO || mode > CCUBE_TRANSPORT_PULL
                               ? fail(CCUBE_ERR_INVALID_ARG, "transport %d out of range", mode)
                               : CCUBE_SUCCESS;
  CC_TRY(agree_setting("transport", mode, v));
  if (mode == g.transport) return CCUBE_SUCCESS;
  CUDA_TRY(cudaDeviceSynchronize());
  g.transport = mode;
  for (auto &kv : g.tasks) cudaFree(kv.second.d_tasks);
  g.tasks.clear();
  for (auto &R : g.regs) {
    if (!R->recv[0] && needs_recv_planes()) {  // loopback only: planes are local
      for (int i = 0; i < g.nlocal; ++i) CUDA_TRY(cudaMalloc(&R->recv[i], 2 * R->plane));
      R->world_recv.assign(g.world, nullptr);
      for (int i = 0; i < g.nlocal; ++i) R->world_recv[g.rank0 + i] = R->recv[i];
    }
    CC_TRY(build_params(R.get()));
  }
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_set_trace(uint64_t *trace, size_t kmax) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  if (trace && kmax == 0) return fail(CCUBE_ERR_INVALID_ARG, "kmax == 0");
  g.trace = trace;
  g.trace_kmax = trace ? kmax : 0;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_finalize(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g.init) return fail(CCUBE_ERR_NOT_INITIALIZED, "ccube_init has not been called");
  cudaDeviceSynchronize();
  ccube_result_t rc = CCUBE_SUCCESS;
  if (g.nproc > 1) {
    std::vector<int> dummy(g.nproc);
    int one = 1;
    rc = do_allgather(&one, dummy.data(), sizeof(int));
  }
  release_all();
  g = Comm();
  return rc;
}

const char *ccube_last_error(void) { return g_err.c_str(); }

ccube_result_t ccube_get_info(ccube_info_t *info) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!info) return fail(CCUBE_ERR_INVALID_ARG, "info is NULL");
  memset(info, 0, sizeof *info);
  info->initialized = g.init;
  info->world_size = g.world;
  info->rank = g.rank0;
  info->nlocal = g.nlocal;
  info->ntrees = g.ntrees;
  info->channels = g.channels;
  info->threads = g.threads;
  info->overlap = g.overlap;
  info->transport = g.transport;
  info->chunk_bytes = g.chunk_bytes;
  info->epoch_base[0] = g.base[0];
  info->epoch_base[1] = g.base[1];
  info->last_channels = g.last_channels;
  info->last_ctas = g.last_ctas;
  info->datapath = g.datapath;
  info->last_tma = g.last_tma;
  info->protocol = g.ll;
  info->last_ll = g.last_ll;
  info->last_threads = g.last_threads;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_set_placement(const int *perm, int P) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g.init) return fail(CCUBE_ERR_ALREADY_INITIALIZED, "set the placement before ccube_init");
  if (!perm) {
    g_place_P = 0;
    return CCUBE_SUCCESS;
  }
  if (P < 1 || P > CCUBE_MAX_RANKS) return fail(CCUBE_ERR_INVALID_ARG, "bad P %d", P);
  if (!is_permutation(perm, P))
    return fail(CCUBE_ERR_INVALID_ARG, "placement is not a permutation of 0..%d", P - 1);
  for (int v = 0; v < P; ++v) g_place[v] = perm[v];
  g_place_P = P;
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_plan_placement(int P, ccube_tree_kind_t kind, const double *bw, int *perm) {
  if (P < 1 || P > CCUBE_MAX_RANKS || !bw || !perm)
    return fail(CCUBE_ERR_INVALID_ARG, "bad P, bw or perm");
  if (kind != CCUBE_TREE_SINGLE && kind != CCUBE_TREE_DOUBLE && kind != CCUBE_TREE_ROTATED)
    return fail(CCUBE_ERR_INVALID_ARG, "bad tree kind %d", (int)kind);
  if (!plan_placement(P, kind, bw, perm))
    return fail(CCUBE_ERR_UNSUPPORTED, "placement planning supports P <= 8");
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_tree_parents_placed(int P, ccube_tree_kind_t kind, int tree,
                                         const int *perm, int *parent) {
  if (P < 1 || P > kTreeMaxP || !parent) return fail(CCUBE_ERR_INVALID_ARG, "bad P or parent");
  if (kind != CCUBE_TREE_SINGLE && kind != CCUBE_TREE_DOUBLE && kind != CCUBE_TREE_ROTATED)
    return fail(CCUBE_ERR_INVALID_ARG, "bad tree kind %d", (int)kind);
  if (tree < 0 || tree >= num_trees(P, kind))
    return fail(CCUBE_ERR_INVALID_ARG, "bad tree index %d", tree);
  if (perm && (P > CCUBE_MAX_RANKS || !is_permutation(perm, P)))
    return fail(CCUBE_ERR_INVALID_ARG, "placement is not a permutation of 0..%d", P - 1);
  Tree t;
  build_tree(P, kind, tree, &t);
  if (perm) place_tree(perm, &t);
  for (int v = 0; v < P; ++v) parent[v] = t.parent[v];
  return CCUBE_SUCCESS;
}

ccube_result_t ccube_tree_parents(int P, ccube_tree_kind_t kind, int tree, int *parent) {
  if (P < 1 || P > kTreeMaxP || !parent) return fail(CCUBE_ERR_INVALID_ARG, "bad P or parent");
  if (kind != CCUBE_TREE_SINGLE && kind != CCUBE_TREE_DOUBLE && kind != CCUBE_TREE_ROTATED)
    return fail(CCUBE_ERR_INVALID_ARG, "bad tree kind %d", (int)kind);
  if (tree < 0 || tree >= num_trees(P, kind))
    return fail(CCUBE_ERR_INVALID_ARG, "bad tree index %d", tree);
  Tree t;
  build_tree(P, kind, tree, &t);
  for (int v = 0; v < P; ++v) parent[v] = t.parent[v];
  return CCUBE_SUCCESS;
}

}  // extern "C"
