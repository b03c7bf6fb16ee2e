// tree_allreduce.cu — the C-Cube hot path on sm_100a.
//
// One launch per AllReduce call ("one-shot").  Every CTA is one task
// (local rank, tree, role, channel): it owns slice `channel` of every chunk of
// `tree` and walks the tree-local chunks k = 0..K_t-1 in order (the tree keeps
// chunk order, Obs #3 P:L145; the gradient queue relies on it).
//
//   role UP   (a4, reduce-up): once every child's partial of chunk k is
//             available, combine own ⊕ child_lo ⊕ child_hi in that fixed order
//             (R2/R3) and hand the result to the parent (PUSH: 128-bit stores into
//             the parent's receive plane over NVLink; PULL: in place in my own
//             buffer, read by the parent).  The root writes the final value into its
//             own buffer and — in C1 — straight into its children's
//             buffers, publishing their Enqueue Semaphores: the reduce->broadcast
//             turnaround costs no extra pass.
//   role DOWN (a5, broadcast-down): once my Enqueue Semaphore says chunk k landed
//             in my buffer (written there by my parent, Fig 9), copy it into
//             each child's buffer and publish the children's semaphores.  In B mode
//             the root also runs a DOWN task that starts only after all K_t chunks
//             are reduced (Fig 7(a)).
//
// CTA = 1 control warp + W data warps (warp specialisation).  The control warp
// polls the upstream counters (one lane per child, .gpu/.sys acquire), publishes
// "chunks ready" to the data warps through shared memory, collects per-warp
// "chunks done" counters and releases the downstream counters (fence + one relaxed
// store covering every chunk finished so far: counters are monotone and waits are
// ">=", Fig 11 "check").  Data warps never wait on a fence; each streams its share
// of every chunk slice with 128-bit accesses, U vectors in flight per source.
// Every spin has a %globaltimer watchdog (CCUBE_WATCHDOG_MS).
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace ccube {
namespace {

constexpr int kMaxThreads = 288;  // up to 8 data warps + the control warp
constexpr int kMaxDataWarps = 8;
constexpr int kMinBlocksPerSm = 2;  // two CTAs per SM: <= 112 registers per thread

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

template <bool SYS>
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t *p) {
  uint64_t v;
  if (SYS)
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  else
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

template <bool SYS>
__device__ __forceinline__ void fence_release() {
  if (SYS)
    asm volatile("fence.acq_rel.sys;" ::: "memory");
  else
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

template <bool SYS>
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
  if (SYS)
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t warp_min(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t w = __shfl_xor_sync(0xffffffffu, v, o);
    v = w < v ? w : v;
  }
  return v;
}

// Watchdog bookkeeping for the control warp.
struct Watch {
  uint64_t last;       // time of the last progress
  uint64_t next_err;   // next time to look at the host error word
  uint32_t spins;
};

__device__ __forceinline__ void watch_reset(Watch &w) {
  w.last = globaltimer();
  w.next_err = w.last + 1000000ull;
  w.spins = 0;
}

// true = keep going; false = abort (timeout here or error elsewhere)
__device__ __forceinline__ bool watch_tick(Watch &w, const LaunchArgs &a, uint64_t target,
                                           uint64_t seen) {
  if (++w.spins & 63) return true;
  const uint64_t now = globaltimer();
  if (now < w.next_err) return true;
  w.next_err = now + 1000000ull;
  if (*reinterpret_cast<volatile int *>(a.err) != 0) return false;
  if (now - w.last > a.timeout_ns) {
    volatile int *e = reinterpret_cast<volatile int *>(a.err);
    e[1] = static_cast<int>(blockIdx.x);
    e[2] = static_cast<int>(target & 0x7fffffff);
    e[3] = static_cast<int>(seen & 0x7fffffff);
    __threadfence_system();
    e[0] = 1;  // 1 = watchdog timeout
    __threadfence_system();
    return false;
  }
  return true;
}

// ---- element combine (R2/R3) ------------------------------------------------
__device__ __forceinline__ float bf_lo(uint32_t w) { return __uint_as_float(w << 16); }
__device__ __forceinline__ float bf_hi(uint32_t w) { return __uint_as_float(w & 0xffff0000u); }
__device__ __forceinline__ uint32_t bf_round(float f) {
  return static_cast<uint32_t>(__bfloat16_as_ushort(__float2bfloat16_rn(f)));
}

template <int DT>
struct Combine;

template <>
struct Combine<kInt32> {
  template <int N>
  __device__ __forceinline__ static uint4 vec(const uint4 (&v)[N]) {
    uint4 r = v[0];
#pragma unroll
    for (int i = 1; i < N; ++i) {  // two's complement wrap
      r.x += v[i].x; r.y += v[i].y; r.z += v[i].z; r.w += v[i].w;
    }
    return r;
  }
  template <int N>
  __device__ __forceinline__ static void scalar(const char *const *src, char *const *dst,
                                                int nout, uint64_t e) {
    uint32_t r = reinterpret_cast<const uint32_t *>(src[0])[e];
#pragma unroll
    for (int i = 1; i < N; ++i) r += reinterpret_cast<const uint32_t *>(src[i])[e];
    for (int d = 0; d < nout; ++d) reinterpret_cast<uint32_t *>(dst[d])[e] = r;
  }
};

template <>
struct Combine<kFloat32> {
  __device__ __forceinline__ static uint32_t add(uint32_t a, uint32_t b) {
    return __float_as_uint(__fadd_rn(__uint_as_float(a), __uint_as_float(b)));
  }
  template <int N>
  __device__ __forceinline__ static uint4 vec(const uint4 (&v)[N]) {
    uint4 r = v[0];
#pragma unroll
    for (int i = 1; i < N; ++i) {  // left to right, IEEE RN, no contraction
      r.x = add(r.x, v[i].x); r.y = add(r.y, v[i].y);
      r.z = add(r.z, v[i].z); r.w = add(r.w, v[i].w);
    }
    return r;
  }
  template <int N>
  __device__ __forceinline__ static void scalar(const char *const *src, char *const *dst,
                                                int nout, uint64_t e) {
    uint32_t r = reinterpret_cast<const uint32_t *>(src[0])[e];
#pragma unroll
    for (int i = 1; i < N; ++i) r = add(r, reinterpret_cast<const uint32_t *>(src[i])[e]);
    for (int d = 0; d < nout; ++d) reinterpret_cast<uint32_t *>(dst[d])[e] = r;
  }
};

template <>
struct Combine<kBFloat16> {
  // widen to fp32, add in the fixed order, round ONCE per node output (RNE)
  template <int N>
  __device__ __forceinline__ static uint32_t word(const uint32_t (&w)[N]) {
    float lo = bf_lo(w[0]), hi = bf_hi(w[0]);
#pragma unroll
    for (int i = 1; i < N; ++i) {
      lo = __fadd_rn(lo, bf_lo(w[i]));
      hi = __fadd_rn(hi, bf_hi(w[i]));
    }
    return bf_round(lo) | (bf_round(hi) << 16);
  }
  template <int N>
  __device__ __forceinline__ static uint4 vec(const uint4 (&v)[N]) {
    if constexpr (N == 1) {
      return v[0];  // a leaf forwards its own bits untouched
    } else {
      uint32_t a[N], b[N], c[N], d[N];
#pragma unroll
      for (int i = 0; i < N; ++i) { a[i] = v[i].x; b[i] = v[i].y; c[i] = v[i].z; d[i] = v[i].w; }
      return make_uint4(word<N>(a), word<N>(b), word<N>(c), word<N>(d));
    }
  }
  template <int N>
  __device__ __forceinline__ static void scalar(const char *const *src, char *const *dst,
                                                int nout, uint64_t e) {
    uint16_t r = reinterpret_cast<const uint16_t *>(src[0])[e];
    if (N > 1) {
      float f = __uint_as_float(static_cast<uint32_t>(r) << 16);
#pragma unroll
      for (int i = 1; i < N; ++i)
        f = __fadd_rn(f, __uint_as_float(
                             static_cast<uint32_t>(reinterpret_cast<const uint16_t *>(src[i])[e])
                             << 16));
      r = static_cast<uint16_t>(bf_round(f));
    }
    for (int d = 0; d < nout; ++d) reinterpret_cast<uint16_t *>(dst[d])[e] = r;
  }
};

__device__ __forceinline__ void trace_landing(const LaunchArgs &a, int local, int t, uint32_t k0,
                                              uint32_t k1, int j) {
  if (a.trace == nullptr || local < 0) return;
  const uint64_t now = globaltimer();
  for (uint32_t k = k0; k < k1 && k < a.trace_kmax; ++k) {
    const uint64_t idx =
        ((static_cast<uint64_t>(local) * a.ntrees + t) * a.trace_kmax + k) * a.nchannels + j;
    a.trace[idx] = now;
  }
}

// ---- TMA staging primitives ----------------------------------------------------------
constexpr int kStages = 4;                 // ring depth (per CTA)
constexpr int kMaxIn = 1 + kMaxChildren;   // sources of a combine

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
               : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {  // .release.cta
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ bool mbar_test(uint64_t *bar, uint32_t parity) {  // .acquire.cta
  uint32_t ok;
  asm volatile(
      "{ .reg .pred p; mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2; "
      "selp.u32 %0, 1, 0, p; }"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}

// blocking wait that gives up when the producer aborted
__device__ __forceinline__ bool mbar_wait(uint64_t *bar, uint32_t parity, const int *abort) {
  uint32_t spins = 0;
  while (true) {
    uint32_t ok;
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; "
        "selp.u32 %0, 1, 0, p; }"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    if (ok) return true;
    if ((++spins & 15) == 0 && *reinterpret_cast<const volatile int *>(abort)) return false;
  }
}

__device__ __forceinline__ void bulk_load(void *smem_dst, const void *gmem_src, uint32_t bytes,
                                          uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(smem_dst)),
      "l"(gmem_src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// ---- segment geometry --------------------------------------------------------------
// A CTA's work for (tree t, channel j) is slice j of every tree-local chunk, cut
// into segments (TMA path) or blocks (LSU path) of `seg` bytes, taken in order.
// Channel slices are made of whole kUnit-byte units: channel j owns units
// [j*n/J, (j+1)*n/J) of the n units of a chunk, so every slice (except at the
// chunk end) is a multiple of the LSU block size and no lane idles.
constexpr uint32_t kUnit = 2048;

struct SegMap {
  uint64_t chunk_stride;  // bytes between consecutive tree-local chunks (T * E_b)
  uint64_t first;         // byte offset of slice j of tree-local chunk 0
  uint32_t seg;           // segment bytes
  uint32_t nseg;          // segments per full slice
  uint32_t kfull;         // tree-local chunks with a full-length slice
  uint32_t sl_full;       // bytes of a full slice of this channel
  uint32_t nseg_last;     // segments of the short last chunk, incl. a ragged one
  uint32_t last_len;      // bytes of the last chunk's slice (may end off a 16 B boundary)
  uint32_t total;         // kfull * nseg + nseg_last
};

template <int ES>
__device__ __forceinline__ SegMap seg_map(const LaunchArgs &a, int t, int j, uint32_t seg) {
  SegMap m;
  const uint64_t Eb = static_cast<uint64_t>(a.elems_per_chunk) * ES;
  const uint32_t nunits = static_cast<uint32_t>((Eb + kUnit - 1) / kUnit);  // Eb < 2^31
  const uint64_t lo = static_cast<uint64_t>(j * nunits / a.nchannels) * kUnit;
  const uint64_t hi = min(static_cast<uint64_t>((j + 1) * nunits / a.nchannels) * kUnit, Eb);
  m.seg = seg;
  m.chunk_stride = Eb * a.ntrees;
  m.first = static_cast<uint64_t>(t) * Eb + lo;
  m.sl_full = static_cast<uint32_t>(hi > lo ? hi - lo : 0);
  m.nseg = (m.sl_full + m.seg - 1) / m.seg;
  const uint32_t K = a.K[t];
  const uint64_t nbytes = a.count * ES;
  const uint64_t Ktot = (a.count + a.elems_per_chunk - 1) / a.elems_per_chunk;
  const uint64_t C = Ktot - 1;  // last global chunk
  m.kfull = K;
  m.last_len = 0;
  m.nseg_last = 0;
  if (K > 0 && (C % a.ntrees) == static_cast<uint64_t>(t) && nbytes < (C + 1) * Eb) {
    m.kfull = K - 1;  // this tree carries the short last chunk
    const uint64_t s0 = C * Eb + lo;
    m.last_len = static_cast<uint32_t>(s0 < nbytes ? min(static_cast<uint64_t>(m.sl_full), nbytes - s0) : 0);
    const uint32_t aligned = m.last_len & ~15u;
    m.nseg_last = (aligned + m.seg - 1) / m.seg + ((m.last_len & 15u) ? 1 : 0);
  }
  m.total = m.nseg ? m.kfull * m.nseg + m.nseg_last : m.nseg_last;
  return m;
}

__device__ __forceinline__ uint32_t seg_chunk(const SegMap &m, uint32_t G) {
  if (m.nseg == 0) return m.kfull;
  const uint32_t k = G / m.nseg;
  return k < m.kfull ? k : m.kfull;
}

// byte offset in the buffer and length of segment G; len < 16 marks the ragged
// sub-vector tail at the very end of the buffer (scalar path, no TMA)
__device__ __forceinline__ void seg_range(const SegMap &m, uint32_t G, uint64_t *off,
                                          uint32_t *len) {
  const uint32_t k = seg_chunk(m, G);
  const uint32_t s = G - k * m.nseg;
  const uint64_t base = m.first + static_cast<uint64_t>(k) * m.chunk_stride;
  if (k < m.kfull) {
    *off = base + static_cast<uint64_t>(s) * m.seg;
    *len = min(m.seg, m.sl_full - s * m.seg);
    return;
  }
  const uint32_t aligned = m.last_len & ~15u;
  const uint32_t full_segs = (aligned + m.seg - 1) / m.seg;
  if (s < full_segs) {
    *off = base + static_cast<uint64_t>(s) * m.seg;
    *len = min(m.seg, aligned - s * m.seg);
  } else {
    *off = base + aligned;
    *len = m.last_len - aligned;  // 1..15 bytes
  }
}

// Incremental form of seg_chunk/seg_range for a warp that takes every W-th block.
struct BlockIter {
  uint32_t G;    // block index
  uint32_t k;    // its chunk (tree-local)
  uint32_t s;    // its segment inside the chunk slice
  uint64_t off;  // byte offset in the buffer
  uint32_t len;  // bytes (< 16: ragged buffer end)
};

__device__ __forceinline__ void block_fill(const SegMap &m, BlockIter &it) {
  if (it.G >= m.total) return;
  const uint64_t base = m.first + static_cast<uint64_t>(it.k) * m.chunk_stride;
  if (it.k < m.kfull) {
    it.off = base + static_cast<uint64_t>(it.s) * m.seg;
    it.len = min(m.seg, m.sl_full - it.s * m.seg);
    return;
  }
  const uint32_t aligned = m.last_len & ~15u;
  const uint32_t full_segs = (aligned + m.seg - 1) / m.seg;
  if (it.s < full_segs) {
    it.off = base + static_cast<uint64_t>(it.s) * m.seg;
    it.len = min(m.seg, aligned - it.s * m.seg);
  } else {
    it.off = base + aligned;
    it.len = m.last_len - aligned;
  }
}

__device__ __forceinline__ BlockIter block_iter(const SegMap &m, uint32_t G) {
  BlockIter it;
  it.G = G;
  it.k = seg_chunk(m, G);
  it.s = G - it.k * m.nseg;
  it.off = 0;
  it.len = 0;
  block_fill(m, it);
  return it;
}

__device__ __forceinline__ void block_next(const SegMap &m, BlockIter &it, uint32_t W) {
  it.G += W;
  it.s += W;
  while (it.k < m.kfull && it.s >= m.nseg) {  // full chunks: nseg segments each
    it.s -= m.nseg;
    ++it.k;
  }
  block_fill(m, it);
}

// Sources and destinations of a task (a4/a5/a6).
struct Endpoints {
  const char *src[kMaxIn];
  char *dst[kMaxIn];
  int nin, nout;
};

__device__ __forceinline__ Endpoints endpoints(const LaunchArgs &a, const TreeParams &p, int role) {
  Endpoints e;
  if (role == kRoleUp) {
    e.nin = 1 + p.nchild;
    for (int q = 0; q < e.nin; ++q) e.src[q] = p.up_src[q];
    e.dst[0] = p.up_dst;
    e.nout = 1;
    if (p.is_root && a.overlap) {  // C1 turnaround: final straight into the children
      for (int s = 0; s < p.nchild; ++s) e.dst[1 + s] = p.child_buf[s];
      e.nout += p.nchild;
    }
  } else {
    e.nin = 1;
    e.src[0] = p.buf;
    for (int s = 0; s < p.nchild; ++s) e.dst[s] = p.child_buf[s];
    e.nout = p.nchild;
  }
  return e;
}

struct Shared {
  uint64_t full[kStages];   // TMA path: producer -> consumers, stage loaded (complete_tx)
  uint64_t empty[kStages];  // TMA path: consumers -> producer, stage consumed
  uint64_t ready;           // LSU path: chunks whose inputs are available (control -> data)
  uint64_t done[kMaxDataWarps];  // LSU path: chunks finished by data warp w (data -> control)
  int abort;
};

// CTA-scope release/acquire on shared memory (control <-> data warps)
__device__ __forceinline__ void st_release_cta(uint64_t *p, uint64_t v) {
  asm volatile("st.release.cta.shared.u64 [%0], %1;" ::"r"(smem_u32(p)), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_cta(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.cta.shared.u64 %0, [%1];" : "=l"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}

__device__ __forceinline__ char *stage_ptr(char *stages, uint32_t seg, int st, int q) {
  return stages + (static_cast<size_t>(st) * kMaxIn + q) * seg;
}

// ---- control / producer warp -------------------------------------------------------
// Releases chunks [pub, d) downstream: one fence, then one store per counter.
template <bool SYS>
__device__ __forceinline__ void publish(const LaunchArgs &a, const TreeParams &p, int role, int t,
                                        int j, uint32_t pub, uint32_t d, uint64_t base) {
  const int stride = j * kFlagStrideU64;
  const uint64_t v = base + d;
  fence_release<SYS>();
  if (role == kRoleUp && !p.is_root) {
    st_relaxed<SYS>(p.head_out + stride, v);
    return;
  }
  if (role == kRoleUp) {  // root: the chunk is final in my own buffer
    st_relaxed<SYS>(p.enq + stride, v);
    trace_landing(a, p.self_local, t, pub, d, j);
    if (!a.overlap) return;
  }
  for (int s = 0; s < p.nchild; ++s) {  // root in C1, or any DOWN task
    st_relaxed<SYS>(p.child_enq[s] + stride, v);
    trace_landing(a, p.child_local[s], t, pub, d, j);
  }
}

// Leaf completion: the kernel completes only once the whole result has landed.
template <bool SYS>
__device__ __forceinline__ void leaf_wait(const LaunchArgs &a, const TreeParams &p, int role,
                                          int t, int j) {
  const int stride = j * kFlagStrideU64;
  const uint64_t target = a.base[t] + a.K[t];
  if (role == kRoleUp && !p.is_root && p.nchild == 0 && (threadIdx.x & 31) == 0) {
    Watch wd;
    watch_reset(wd);
    while (ld_acquire<SYS>(p.enq + stride) < target) {
      if (!watch_tick(wd, a, target, 0)) {
        st_relaxed<SYS>(p.enq + stride, ~0ull);
        return;
      }
    }
  }
}

template <int ES, bool SYS>
__device__ void control_warp_tma(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                                 Shared &sh, char *stages) {
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const uint64_t base = a.base[t];
  const int stride = j * kFlagStrideU64;
  const Endpoints e = endpoints(a, p, role);
  const SegMap m = seg_map<ES>(a, t, j, a.seg_bytes);
  // upstream counters: UP waits on each child's head, DOWN on my own semaphore
  const uint64_t *up = nullptr;
  if (role == kRoleUp) {
    if (lane < p.nchild) up = p.head_in[lane] + stride;
  } else if (lane == 0) {
    up = p.enq + stride;
  }
  const bool hold_all = role == kRoleDown && p.is_root;  // B-mode root (Obs #1)
  uint64_t ready = (role == kRoleUp && p.nchild == 0) ? K : 0;  // a leaf's input is ready
  bool fresh = true;  // ready advanced since the last proxy fence
  uint32_t issued = 0, retired = 0, pub = 0;
  Watch wd;
  watch_reset(wd);
  while (pub < K) {
    bool moved = false;
    // (1) readiness: poll upstream (one lane per child, .gpu/.sys acquire)
    const uint32_t need = issued < m.total ? seg_chunk(m, issued) : K;
    if (ready < K && need >= ready) {
      uint64_t v = up ? ld_acquire<SYS>(up) : ~0ull;
      v = warp_min(v);
      uint64_t r = v > base ? v - base : 0;
      if (r > K) r = K;
      if (hold_all && r < K) r = 0;
      if (r > ready) {
        __syncwarp();  // every lane's acquire is ordered before lane 0's TMA issue
        ready = r;
        fresh = true;
        moved = true;
      }
    }
    // (2) issue TMA loads for ready segments into free stages
    if (lane == 0) {
      while (issued < m.total && issued - retired < kStages) {
        const uint32_t k = seg_chunk(m, issued);
        if (k >= ready) break;
        if (fresh) {  // generic-proxy acquire -> async-proxy (TMA) reads
          asm volatile("fence.proxy.async.global;" ::: "memory");
          fresh = false;
        }
        uint64_t off;
        uint32_t len;
        seg_range(m, issued, &off, &len);
        const int st = issued % kStages;
        if (len >= 16) {
          mbar_expect_tx(&sh.full[st], len * e.nin);
          for (int q = 0; q < e.nin; ++q)
            bulk_load(stage_ptr(stages, m.seg, st, q), e.src[q] + off, len, &sh.full[st]);
        } else {
          mbar_arrive(&sh.full[st]);  // ragged tail: consumers read it from global
        }
        ++issued;
        moved = true;
      }
      // (3) retire stages the consumers have finished (non-blocking)
      while (retired < issued && mbar_test(&sh.empty[retired % kStages], (retired / kStages) & 1)) {
        ++retired;
        moved = true;
      }
    }
    issued = __shfl_sync(0xffffffffu, issued, 0);
    retired = __shfl_sync(0xffffffffu, retired, 0);
    fresh = __shfl_sync(0xffffffffu, fresh, 0);
    // (4) a chunk is done once every segment of it is retired
    const uint32_t d = retired < m.total ? seg_chunk(m, retired) : K;
    if (d > pub) {
      if (lane == 0) publish<SYS>(a, p, role, t, j, pub, d, base);
      pub = d;
      moved = true;
    }
    if (moved) {
      watch_reset(wd);
    } else if (!watch_tick(wd, a, base + ready + 1, base + pub)) {
      if (lane == 0) {
        *reinterpret_cast<volatile int *>(&sh.abort) = 1;
        st_relaxed<SYS>(p.enq + stride, ~0ull);  // release gradient-queue waiters
      }
      return;
    }
  }
  leaf_wait<SYS>(a, p, role, t, j);
}

// A leaf on a PULL edge: its input already sits where the parent reads it.  One
// warp publishes every channel's head at once and waits for the result.
template <bool SYS>
__device__ void pulled_leaf(const LaunchArgs &a, const TreeParams &p, int t) {
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const uint64_t base = a.base[t];
  fence_release<SYS>();
  for (int j = lane; j < static_cast<int>(a.nchannels); j += 32)
    st_relaxed<SYS>(p.head_out + j * kFlagStrideU64, base + K);
  for (int j = lane; j < static_cast<int>(a.nchannels); j += 32) {
    Watch wd;
    watch_reset(wd);
    while (ld_acquire<SYS>(p.enq + j * kFlagStrideU64) < base + K) {
      if (!watch_tick(wd, a, base + K, 0)) {
        st_relaxed<SYS>(p.enq + j * kFlagStrideU64, ~0ull);
        break;
      }
    }
  }
}

// ---- consumer (data) warps -----------------------------------------------------------
template <int DT, int NIN>
__device__ __forceinline__ void combine_stage(char *stages, uint32_t seg, int st, uint32_t len,
                                              char *const *dst, int nout, uint64_t off, int w,
                                              int W) {
  const int lane = threadIdx.x & 31;
  const char *b = stage_ptr(stages, seg, st, 0);
  for (uint32_t v = w * 32 + lane; v < len / 16; v += W * 32) {
    uint4 x[NIN];
#pragma unroll
    for (int q = 0; q < NIN; ++q)
      x[q] = *reinterpret_cast<const uint4 *>(b + static_cast<size_t>(q) * seg + v * 16);
    const uint4 r = Combine<DT>::template vec<NIN>(x);
    for (int d = 0; d < nout; ++d) *reinterpret_cast<uint4 *>(dst[d] + off + v * 16) = r;
  }
}

template <int DT>
__device__ __forceinline__ void combine_scalar(const char *const *src, int nin, char *const *dst,
                                               int nout, uint64_t off, uint32_t len) {
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  const int lane = threadIdx.x & 31;
  const char *ss[kMaxIn];
  char *dd[kMaxIn];
  for (int q = 0; q < nin; ++q) ss[q] = src[q] + off;
  for (int q = 0; q < nout; ++q) dd[q] = dst[q] + off;
  for (uint32_t x = lane; x < len / ES; x += 32) {
    switch (nin) {
      case 1: Combine<DT>::template scalar<1>(ss, dd, nout, x); break;
      case 2: Combine<DT>::template scalar<2>(ss, dd, nout, x); break;
      default: Combine<DT>::template scalar<3>(ss, dd, nout, x); break;
    }
  }
}

template <int DT>
__device__ void data_warp_tma(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                              int w, int W, Shared &sh, char *stages) {
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  const int lane = threadIdx.x & 31;
  const Endpoints e = endpoints(a, p, role);
  const SegMap m = seg_map<ES>(a, t, j, a.seg_bytes);
  for (uint32_t G = 0; G < m.total; ++G) {
    const int st = G % kStages;
    if (!mbar_wait(&sh.full[st], (G / kStages) & 1, &sh.abort)) return;
    uint64_t off;
    uint32_t len;
    seg_range(m, G, &off, &len);
    if (len >= 16) {
      switch (e.nin) {
        case 1: combine_stage<DT, 1>(stages, m.seg, st, len, e.dst, e.nout, off, w, W); break;
        case 2: combine_stage<DT, 2>(stages, m.seg, st, len, e.dst, e.nout, off, w, W); break;
        default: combine_stage<DT, 3>(stages, m.seg, st, len, e.dst, e.nout, off, w, W); break;
      }
    } else if (w == 0) {
      combine_scalar<DT>(e.src, e.nin, e.dst, e.nout, off, len);
    }
    __syncwarp();  // all lanes done with the stage and their stores issued
    if (lane == 0) mbar_arrive(&sh.empty[st]);
  }
}

// ---- LSU path (default): register-staged data warps ------------------------------
// The control warp polls upstream and publishes "chunks ready" in shared memory;
// each data warp streams its items — 16-byte vectors w*32+lane, stepping W*32,
// across the concatenated slices of all chunks — in rounds of U vectors per
// lane per source.  A round may span chunk boundaries (it only needs every lane's
// chunk to be ready), so loads stay in flight across chunks; per-warp "done"
// counters (the chunk of the warp's next item) let the control warp publish
// downstream.
template <bool SYS>
__device__ void control_warp_lsu(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                                 int W, Shared &sh) {
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const uint64_t base = a.base[t];
  const int stride = j * kFlagStrideU64;
  const uint64_t *up = nullptr;
  if (role == kRoleUp) {
    if (lane < p.nchild) up = p.head_in[lane] + stride;
  } else if (lane == 0) {
    up = p.enq + stride;
  }
  const bool hold_all = role == kRoleDown && p.is_root;  // B-mode root (Obs #1)
  uint64_t ready = (role == kRoleUp && p.nchild == 0) ? K : 0;  // a leaf's input is ready
  if (lane == 0) st_release_cta(&sh.ready, ready);
  uint32_t pub = 0;
  Watch wd;
  watch_reset(wd);
  while (pub < K) {
    bool moved = false;
    if (ready < K) {
      uint64_t v = up ? ld_acquire<SYS>(up) : ~0ull;
      v = warp_min(v);
      uint64_t r = v > base ? v - base : 0;
      if (r > K) r = K;
      if (hold_all && r < K) r = 0;
      if (r > ready) {
        __syncwarp();  // every lane's acquire happens before lane 0's release below
        ready = r;
        if (lane == 0) st_release_cta(&sh.ready, ready);
        moved = true;
      }
    }
    uint64_t d = lane < W ? ld_acquire_cta(&sh.done[lane]) : ~0ull;
    d = warp_min(d);
    if (d > pub) {
      __syncwarp();
      if (lane == 0) publish<SYS>(a, p, role, t, j, pub, static_cast<uint32_t>(d), base);
      pub = static_cast<uint32_t>(d);
      moved = true;
    }
    if (moved) {
      watch_reset(wd);
    } else if (!watch_tick(wd, a, base + ready + 1, base + pub)) {
      if (lane == 0) {
        *reinterpret_cast<volatile int *>(&sh.abort) = 1;
        st_relaxed<SYS>(p.enq + stride, ~0ull);  // release gradient-queue waiters
      }
      return;
    }
  }
  leaf_wait<SYS>(a, p, role, t, j);
}

// One data warp's stream: blocks G = w, w+W, ... of 32*U vectors (512*U bytes).
// A block lies inside one chunk's slice, so the readiness check and the base
// address are warp-uniform; lane l handles vectors l + 32u, u < U.
template <int DT, int NIN, int NOUT, int U>
__device__ void lsu_stream(const LaunchArgs &a, const Endpoints &e, int t, int j, int w, int W,
                           Shared &sh) {
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const SegMap m = seg_map<ES>(a, t, j, 512u * U);
  uint64_t ready = 0;
  uint32_t done_reported = 0;
  // Block iterator: this warp's blocks G = w, w+W, ... as (chunk k, segment s),
  // advanced without divisions so the next addresses are ready as soon as the
  // current loads are issued (the loop is load-latency bound).
  BlockIter it = block_iter(m, w);
  while (it.k < K && it.G < m.total) {
    const uint32_t k = it.k;
    if (k >= ready) {
      uint64_t r = 0;
      if (lane == 0) {
        do {
          r = ld_acquire_cta(&sh.ready);
        } while (r <= k && !*reinterpret_cast<volatile int *>(&sh.abort));
      }
      r = __shfl_sync(0xffffffffu, r, 0);
      if (r <= k) return;  // aborted
      ready = r;
    }
    const uint64_t off = it.off;
    const uint32_t len = it.len;
    if (len >= 16) {
      const uint32_t nvec = len / 16;
      uint4 x[U][NIN];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (lane + 32u * u < nvec) {
#pragma unroll
          for (int q = 0; q < NIN; ++q)
            x[u][q] = __ldcg(reinterpret_cast<const uint4 *>(e.src[q] + off + lane * 16 + 512u * u));
        }
      }
      block_next(m, it, W);  // overlaps the loads
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (lane + 32u * u < nvec) {
          const uint4 r = Combine<DT>::template vec<NIN>(x[u]);
#pragma unroll
          for (int q = 0; q < NOUT; ++q)
            *reinterpret_cast<uint4 *>(e.dst[q] + off + lane * 16 + 512u * u) = r;
        }
      }
    } else {
      combine_scalar<DT>(e.src, NIN, e.dst, NOUT, off, len);  // ragged end of the buffer
      block_next(m, it, W);
    }
    const uint32_t d = it.G < m.total ? it.k : K;
    if (d > done_reported) {
      __syncwarp();  // every lane's stores precede the release
      if (lane == 0) st_release_cta(&sh.done[w], d);
      done_reported = d;
    }
  }
  if (done_reported < K) {
    __syncwarp();
    if (lane == 0) st_release_cta(&sh.done[w], K);
  }
}

template <int DT, int NIN>
__device__ __forceinline__ void lsu_nout(const LaunchArgs &a, const Endpoints &e, int t, int j,
                                         int w, int W, Shared &sh) {
  constexpr int U = NIN == 1 ? 8 : 4;  // block = 4 KB (copies) or 2 KB (combines)
  switch (e.nout) {
    case 1: lsu_stream<DT, NIN, 1, U>(a, e, t, j, w, W, sh); break;
    case 2: lsu_stream<DT, NIN, 2, U>(a, e, t, j, w, W, sh); break;
    default: lsu_stream<DT, NIN, 3, U>(a, e, t, j, w, W, sh); break;
  }
}

template <int DT>
__device__ void data_warp_lsu(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                              int w, int W, Shared &sh) {
  const Endpoints e = endpoints(a, p, role);
  if (e.nout == 0) {  // nothing to write (cannot happen for scheduled tasks)
    if ((threadIdx.x & 31) == 0) st_release_cta(&sh.done[w], a.K[t]);
    return;
  }
  switch (e.nin) {
    case 1: lsu_nout<DT, 1>(a, e, t, j, w, W, sh); break;
    case 2: lsu_nout<DT, 2>(a, e, t, j, w, W, sh); break;
    default: lsu_nout<DT, 3>(a, e, t, j, w, W, sh); break;
  }
}

// ---- ASYNC path (default): per-lane cp.async rings ------------------------------
// Same work split as the LSU path (warp w takes blocks G = w, w+W, ... of 32*kAU
// vectors), but every lane stages ITS OWN 16-byte vectors of up to kRing/NIN
// blocks ahead through shared memory with cp.async (LDGSTS): loads stay in flight
// without holding registers, so each warp keeps ~12 KB of reads outstanding
// continuously instead of one register round at a time.  A lane only ever reads
// back what it copied itself, so cp.async.wait_group alone orders the data (no
// barrier, no cross-proxy fence).  Readiness is checked per block before its loads
// are issued, exactly as in the LSU path.
constexpr int kAU = 2;                       // vectors per lane per source per block
constexpr uint32_t kABlock = 512u * kAU;     // bytes per source per block (1 KB)
constexpr int kRing = 12;                    // source-blocks in flight per warp
constexpr uint32_t kRingBytes = kRing * kABlock;  // shared memory per data warp

__device__ __forceinline__ void cp_async16(uint32_t smem, const void *gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() {
  asm volatile("cp.async.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
// wait until at most `pending` (0 <= pending < S) groups are outstanding
template <int S>
__device__ __forceinline__ void cp_async_wait_dyn(uint32_t pending) {
  if constexpr (S > 1) {
    if (pending >= S - 1) {
      cp_async_wait<S - 1>();
      return;
    }
    cp_async_wait_dyn<S - 1>(pending);
  } else {
    cp_async_wait<0>();
  }
}

template <int DT, int NIN, int NOUT>
__device__ void async_stream(const LaunchArgs &a, const Endpoints &e, int t, int j, int w, int W,
                             Shared &sh, char *ring) {
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  constexpr int S = kRing / NIN;  // blocks in flight
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const SegMap m = seg_map<ES>(a, t, j, kABlock);
  const uint32_t nb = m.total > static_cast<uint32_t>(w) ? (m.total - w + W - 1) / W : 0;
  const uint32_t my = smem_u32(ring) + lane * 16;
  uint64_t ready = 0;
  uint32_t issued = 0, done_reported = 0;
  for (uint32_t i = 0; i < nb; ++i) {
    // top up: issue the loads of blocks i .. i+S-1 that are ready
    while (issued < nb && issued < i + S) {
      const uint32_t G = w + issued * W;
      const uint32_t k = seg_chunk(m, G);
      if (k >= ready) {
        uint64_t r = 0;
        if (lane == 0) {
          r = ld_acquire_cta(&sh.ready);
          if (issued == i)  // nothing in flight to work on: wait for it
            while (r <= k && !*reinterpret_cast<volatile int *>(&sh.abort))
              r = ld_acquire_cta(&sh.ready);
        }
        r = __shfl_sync(0xffffffffu, r, 0);
        if (r > ready) ready = r;
        if (k >= ready) {
          if (issued == i) return;  // aborted
          break;                    // work on what is in flight, re-check later
        }
      }
      uint64_t off;
      uint32_t len;
      seg_range(m, G, &off, &len);
      const uint32_t st = (issued % S) * NIN * kABlock;
      if (len >= 16) {
        const uint32_t nvec = len / 16;
#pragma unroll
        for (int u = 0; u < kAU; ++u)
          if (lane + 32u * u < nvec) {
#pragma unroll
            for (int q = 0; q < NIN; ++q)
              cp_async16(my + st + q * kABlock + 512u * u, e.src[q] + off + lane * 16 + 512u * u);
          }
      }
      cp_async_commit();  // one group per block (empty for the ragged tail)
      ++issued;
    }
    cp_async_wait_dyn<S>(issued - i - 1);
    const uint32_t G = w + i * W;
    uint64_t off;
    uint32_t len;
    seg_range(m, G, &off, &len);
    if (len >= 16) {
      const uint32_t nvec = len / 16;
      const char *stage = ring + (i % S) * NIN * kABlock + lane * 16;
#pragma unroll
      for (int u = 0; u < kAU; ++u) {
        if (lane + 32u * u < nvec) {
          uint4 x[NIN];
#pragma unroll
          for (int q = 0; q < NIN; ++q)
            x[q] = *reinterpret_cast<const uint4 *>(stage + q * kABlock + 512u * u);
          const uint4 r = Combine<DT>::template vec<NIN>(x);
#pragma unroll
          for (int q = 0; q < NOUT; ++q)
            *reinterpret_cast<uint4 *>(e.dst[q] + off + lane * 16 + 512u * u) = r;
        }
      }
    } else {
      combine_scalar<DT>(e.src, NIN, e.dst, NOUT, off, len);  // ragged end of the buffer
    }
    const uint32_t d = i + 1 < nb ? seg_chunk(m, G + W) : K;
    if (d > done_reported) {
      __syncwarp();  // every lane's stores precede the release
      if (lane == 0) st_release_cta(&sh.done[w], d);
      done_reported = d;
    }
  }
  if (done_reported < K) {
    __syncwarp();
    if (lane == 0) st_release_cta(&sh.done[w], K);
  }
}

template <int DT, int NIN>
__device__ __forceinline__ void async_nout(const LaunchArgs &a, const Endpoints &e, int t, int j,
                                           int w, int W, Shared &sh, char *ring) {
  switch (e.nout) {
    case 1: async_stream<DT, NIN, 1>(a, e, t, j, w, W, sh, ring); break;
    case 2: async_stream<DT, NIN, 2>(a, e, t, j, w, W, sh, ring); break;
    default: async_stream<DT, NIN, 3>(a, e, t, j, w, W, sh, ring); break;
  }
}

template <int DT>
__device__ void data_warp_async(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                                int w, int W, Shared &sh, char *stages) {
  const Endpoints e = endpoints(a, p, role);
  char *ring = stages + static_cast<size_t>(w) * kRingBytes;
  if (e.nout == 0) {
    if ((threadIdx.x & 31) == 0) st_release_cta(&sh.done[w], a.K[t]);
    return;
  }
  switch (e.nin) {
    case 1: async_nout<DT, 1>(a, e, t, j, w, W, sh, ring); break;
    case 2: async_nout<DT, 2>(a, e, t, j, w, W, sh, ring); break;
    default: async_nout<DT, 3>(a, e, t, j, w, W, sh, ring); break;
  }
}

template <int DT, bool SYS>
__global__ void __launch_bounds__(kMaxThreads, kMinBlocksPerSm) tree_allreduce_kernel(const LaunchArgs a) {
  __shared__ Shared sh;
  extern __shared__ __align__(128) char stages[];
  const Task task = a.tasks[blockIdx.x];
  const TreeParams &p = a.params[task.local_rank * a.ntrees + task.tree];
  const int warp = threadIdx.x >> 5;
  if (task.channel == kAllChannels) {
    if (warp == 0) pulled_leaf<SYS>(a, p, task.tree);
    return;
  }
  const int W = (blockDim.x >> 5) - 1;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&sh.full[s], 1);
      mbar_init(&sh.empty[s], W);
    }
    sh.ready = 0;
    sh.abort = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (threadIdx.x < kMaxDataWarps) sh.done[threadIdx.x] = 0;
  __syncthreads();
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  if (a.datapath == kDatapathTma) {
    if (warp == 0)
      control_warp_tma<ES, SYS>(a, p, task.role, task.tree, task.channel, sh, stages);
    else
      data_warp_tma<DT>(a, p, task.role, task.tree, task.channel, warp - 1, W, sh, stages);
  } else if (a.datapath == kDatapathAsync) {
    if (warp == 0)
      control_warp_lsu<SYS>(a, p, task.role, task.tree, task.channel, W, sh);
    else
      data_warp_async<DT>(a, p, task.role, task.tree, task.channel, warp - 1, W, sh, stages);
  } else {
    if (warp == 0)
      control_warp_lsu<SYS>(a, p, task.role, task.tree, task.channel, W, sh);
    else
      data_warp_lsu<DT>(a, p, task.role, task.tree, task.channel, warp - 1, W, sh);
  }
}

struct GateArgs {
  const uint64_t *ctr[kMaxGateCounters];
  uint64_t target[kMaxGateCounters];
  int n;
  int *err;
  uint64_t timeout_ns;
};

// Fallback gradient-queue gate (a9): one warp spins until every counter reaches
// its target; the next kernel on the stream then sees the landed chunks.
template <bool SYS>
__global__ void gate_kernel(const GateArgs g) {
  for (int i = threadIdx.x; i < g.n; i += blockDim.x) {
    const uint64_t t0 = globaltimer();
    while (ld_acquire<SYS>(g.ctr[i]) < g.target[i]) {
      if (globaltimer() - t0 > g.timeout_ns) {
        *reinterpret_cast<volatile int *>(g.err) = 2;  // 2 = gate timeout
        __threadfence_system();
        break;
      }
    }
  }
}

size_t stage_bytes(int datapath, uint32_t seg, int threads) {
  if (datapath == kDatapathTma) return static_cast<size_t>(kStages) * kMaxIn * seg;
  if (datapath == kDatapathAsync) return static_cast<size_t>(threads / 32 - 1) * kRingBytes;
  return 0;
}

template <int DT, bool SYS>
int launch_t(const LaunchArgs &a, int grid, int threads, cudaStream_t s) {
  const size_t smem = stage_bytes(a.datapath, a.seg_bytes, threads);
  cudaError_t e = cudaFuncSetAttribute(tree_allreduce_kernel<DT, SYS>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return static_cast<int>(e);
  tree_allreduce_kernel<DT, SYS><<<grid, threads, smem, s>>>(a);
  return static_cast<int>(cudaGetLastError());
}

template <int DT, bool SYS>
const void *kernel_ptr() {
  return reinterpret_cast<const void *>(tree_allreduce_kernel<DT, SYS>);
}

}  // namespace

int launch_tree_allreduce(const LaunchArgs &args, int dtype, bool sys_scope, int grid,
                          int threads, void *stream) {
  if (threads > kMaxThreads || threads < 64 || threads % 32 ||
      threads / 32 - 1 > kMaxDataWarps || args.seg_bytes < 16 || args.seg_bytes % 16)
    return cudaErrorInvalidValue;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  switch (dtype) {
    case kInt32:
      return sys_scope ? launch_t<kInt32, true>(args, grid, threads, s)
                       : launch_t<kInt32, false>(args, grid, threads, s);
    case kFloat32:
      return sys_scope ? launch_t<kFloat32, true>(args, grid, threads, s)
                       : launch_t<kFloat32, false>(args, grid, threads, s);
    case kBFloat16:
      return sys_scope ? launch_t<kBFloat16, true>(args, grid, threads, s)
                       : launch_t<kBFloat16, false>(args, grid, threads, s);
    default:
      return cudaErrorInvalidValue;
  }
}

int launch_gate(const uint64_t *const *counters, const uint64_t *targets, int n, int *err,
                uint64_t timeout_ns, bool sys_scope, void *stream) {
  if (n <= 0) return cudaSuccess;
  if (n > kMaxGateCounters) return cudaErrorInvalidValue;
  GateArgs g;
  for (int i = 0; i < n; ++i) {
    g.ctr[i] = counters[i];
    g.target[i] = targets[i];
  }
  g.n = n;
  g.err = err;
  g.timeout_ns = timeout_ns;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (sys_scope)
    gate_kernel<true><<<1, 32, 0, s>>>(g);
  else
    gate_kernel<false><<<1, 32, 0, s>>>(g);
  return static_cast<int>(cudaGetLastError());
}

int query_max_blocks_per_sm(int dtype, bool sys_scope, int threads, int datapath,
                            uint32_t seg_bytes, int *blocks) {
  const void *fn = nullptr;
  switch (dtype) {
    case kInt32:
      fn = sys_scope ? kernel_ptr<kInt32, true>() : kernel_ptr<kInt32, false>();
      break;
    case kFloat32:
      fn = sys_scope ? kernel_ptr<kFloat32, true>() : kernel_ptr<kFloat32, false>();
      break;
    default:
      fn = sys_scope ? kernel_ptr<kBFloat16, true>() : kernel_ptr<kBFloat16, false>();
      break;
  }
  const size_t smem = stage_bytes(datapath, seg_bytes, threads);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return static_cast<int>(e);
  return static_cast<int>(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, fn, threads, smem));
}

}  // namespace ccube
