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

#ifndef CCUBE_U_COMBINE
#define CCUBE_U_COMBINE 4  // 16-byte vectors per lane per source in flight (combines)
#endif
#ifndef CCUBE_U_COPY
#define CCUBE_U_COPY 4     // ... (copies; 8 measured 1% slower, v16)
#endif
// Smaller CTAs leave each thread more registers at two CTAs per SM (launch bounds:
// 320 threads -> 96, 256 -> 128, 224 -> 144, 192 -> 168), i.e. room for more
// 16-byte vectors in flight per lane in the combines (the DRAM-reading UP tasks,
// whose bytes in flight set the pipeline's rate).  Per CTA-size bucket:
#ifndef CCUBE_U_COMBINE_S
#define CCUBE_U_COMBINE_S 6    // <= 256 threads (6 data warps + 2 control warps)
#endif
#ifndef CCUBE_U_COMBINE_224
#define CCUBE_U_COMBINE_224 8  // <= 224 threads (5 data warps)
#endif
#ifndef CCUBE_U_COMBINE_192
#define CCUBE_U_COMBINE_192 8  // <= 192 threads (4 data warps)
#endif
#ifndef CCUBE_DONE_INIT
#define CCUBE_DONE_INIT 1  // data warps report their first block's chunk at start
#endif
#ifndef CCUBE_OWN_FIRST
#define CCUBE_OWN_FIRST 1  // combines load their own input before the readiness wait
#endif
#ifndef CCUBE_U_COPY_S
#define CCUBE_U_COPY_S 4
#endif
__host__ __device__ constexpr int u_combine(int maxt) {
  return maxt <= 192 ? CCUBE_U_COMBINE_192
         : maxt <= 224 ? CCUBE_U_COMBINE_224
         : maxt <= 256 ? CCUBE_U_COMBINE_S
                       : CCUBE_U_COMBINE;
}

constexpr int kMaxThreads = 320;  // up to 8 data warps + one or two control warps
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
// Both halves of a word at once: cvt.rn.bf16x2.f32 rounds each input to nearest-even
// exactly as cvt.rn.bf16.f32 does (no FTZ), in one packed conversion (F2FP.PACK_AB)
// instead of two F2F conversions and a byte permute.
__device__ __forceinline__ uint32_t bf_pack(float lo, float hi) {
  uint32_t r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
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
    return bf_pack(lo, hi);
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
                                              uint32_t k1, int j, uint64_t base = 0) {
  if (a.trace == nullptr || local < 0) return;
  const uint64_t now = globaltimer();
  for (uint32_t k = k0; k < k1 && k < a.trace_kmax; ++k) {
    const uint64_t idx =
        ((static_cast<uint64_t>(local) * a.ntrees + t) * a.trace_kmax + k) * a.nchannels + j;
    a.trace[base + idx] = now;
  }
}

constexpr int kMaxIn = 1 + kMaxChildren;  // sources of a combine

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---- chunk / channel geometry (a3) ------------------------------------------------
// Tree-local chunk k of tree t is global chunk g = k*T + t (R4): bytes
// [g*Eb, min((g+1)*Eb, nbytes)).  Its n = ceil(len/kUnit) units are split over the
// J channels, q = n / J each plus one extra unit for r = n % J of them.  WHICH
// channels get the extra unit rotates with k — channel j does iff (j + k) mod J < r —
// so over the whole call every channel streams the same number of bytes to within
// one unit (a static split would leave the channels with q+1 units the critical
// path of every chunk: 4 vs 3.1 units at 256 KiB chunks and 41 channels).  Every
// task of the tree (UP and DOWN, every rank) uses the same split, so the
// per-channel counters describe the same byte ranges on both sides of an edge.
constexpr uint32_t kUnit = 2048;

struct Geo {
  uint64_t Eb;       // chunk bytes
  uint64_t nbytes;   // buffer bytes
  uint64_t stride;   // bytes between consecutive chunks of this tree (T * Eb)
  uint64_t first;    // byte offset of this tree's chunk 0 (t * Eb)
  uint32_t J, j;     // channels, this channel
  uint32_t K;        // tree-local chunks
  uint32_t q, r;     // split of a full chunk's units: q each, one more for r channels
};

struct Slice {
  uint64_t off;  // byte offset in the buffer
  uint32_t len;  // bytes (may end off a 16-byte boundary only at the buffer end)
};

template <int ES>
__device__ __forceinline__ Geo make_geo(const LaunchArgs &a, int t, int j) {
  Geo g;
  g.Eb = static_cast<uint64_t>(a.elems_per_chunk) * ES;
  g.nbytes = a.count * ES;
  g.stride = g.Eb * a.ntrees;
  g.first = g.Eb * t;
  g.J = a.nchannels;
  g.j = j;
  g.K = a.K[t];
  const uint32_t n = static_cast<uint32_t>((g.Eb + kUnit - 1) / kUnit);
  g.q = n / g.J;
  g.r = n % g.J;
  return g;
}

// Slice of channel j in the chunk at byte offset c0, whose tree-local index k has
// c = k mod J.  Channel i gets q units plus one iff (i + c) mod J < r; channel j
// starts after f(c + j) - f(c) extra units, f(x) = #{m < x : m mod J < r}.  With
// c, j < J every term is a compare (no division) except for the short last chunk.
__device__ __forceinline__ Slice slice_at(const Geo &g, uint32_t c, uint64_t c0) {
  const uint64_t clen = min(g.Eb, g.nbytes - c0);
  uint32_t q = g.q, r = g.r;
  if (clen < g.Eb) {  // the short last chunk has its own split
    const uint32_t n = static_cast<uint32_t>((clen + kUnit - 1) / kUnit);
    q = n / g.J;
    r = n % g.J;
  }
  const uint32_t x = c + g.j;                                // < 2J
  const uint32_t fx = x < g.J ? min(x, r) : r + min(x - g.J, r);
  const uint32_t u0 = g.j * q + fx - min(c, r);
  const uint32_t nu = q + ((x < g.J ? x : x - g.J) < r ? 1u : 0u);
  const uint64_t lo = min(static_cast<uint64_t>(u0) * kUnit, clen);
  const uint64_t hi = min(static_cast<uint64_t>(u0 + nu) * kUnit, clen);
  Slice s;
  s.off = c0 + lo;
  s.len = static_cast<uint32_t>(hi - lo);
  return s;
}

// A data warp's walk over its blocks: blocks of `seg` bytes tile each chunk's
// slice; warp w of W takes blocks w, w+W, ... of the concatenation over chunks,
// so a warp's blocks are in chunk order (the readiness check and the base
// address of a block are warp-uniform).  Advanced without divisions.
struct BlockIter {
  uint32_t k;    // chunk (tree-local); K = finished
  uint32_t c;    // k mod J
  uint64_t c0;   // byte offset of chunk k
  uint32_t s;    // block inside the chunk's slice
  uint32_t nb;   // blocks in this chunk's slice
  Slice sl;      // this chunk's slice
};

template <uint32_t SEG>
__device__ __forceinline__ void iter_settle(const Geo &g, BlockIter &it) {
  while (it.k < g.K && it.s >= it.nb) {
    it.s -= it.nb;
    if (++it.k < g.K) {
      it.c = it.c + 1 == g.J ? 0 : it.c + 1;
      it.c0 += g.stride;
      it.sl = slice_at(g, it.c, it.c0);
      it.nb = (it.sl.len + SEG - 1) / SEG;
    }
  }
}

template <uint32_t SEG>
__device__ __forceinline__ BlockIter iter_begin(const Geo &g, uint32_t w) {
  BlockIter it;
  it.k = 0;
  it.c = 0;
  it.c0 = g.first;
  it.s = w;
  it.nb = 0;
  it.sl.off = 0;
  it.sl.len = 0;
  if (g.K > 0) {
    it.sl = slice_at(g, 0, it.c0);
    it.nb = (it.sl.len + SEG - 1) / SEG;
  }
  iter_settle<SEG>(g, it);
  return it;
}

// Sources and destinations of a task (a4/a5/a6).
struct Endpoints {
  const char *src[kMaxIn];
  char *dst[kMaxIn];
  int nin, nout;
  uint32_t keep;  // bit q: dst[q] is re-read later in this launch (L2 evict_last)
  bool sgd;       // this task also applies the fused SGD step to my weights (f2)
  char *w;        // my weights
  const char *gfinal;  // where my final gradient sits (ragged-tail scalar path)
};

// The task that applies rank v's fused SGD step (f2) is the one that handles v's
// final gradient anyway: the root's UP task (it computes it), an interior rank's
// DOWN task (it reads it to forward it), a leaf's UPDATE task.
__device__ __forceinline__ bool does_sgd(const LaunchArgs &a, const TreeParams &p, int role) {
  if (!a.sgd) return false;
  if (role == kRoleUpdate) return true;
  return role == kRoleUp ? p.is_root != 0 : p.is_root == 0;
}

__device__ __forceinline__ Endpoints endpoints(const LaunchArgs &a, const TreeParams &p, int role) {
  Endpoints e;
  e.keep = 0;
  e.sgd = does_sgd(a, p, role);
  e.w = p.w;
  e.gfinal = p.buf;
  if (role == kRoleUpdate) {
    e.nin = 1;
    e.src[0] = p.buf;
    e.nout = 0;
    return e;
  }
  if (role == kRoleUp) {
    e.nin = 1 + p.nchild;
    for (int q = 0; q < e.nin; ++q) e.src[q] = p.up_src[q];
    e.dst[0] = p.up_dst;
    e.nout = 1;
    // a partial is re-read by the parent; the root's final only by its B-mode DOWN task
    if (!p.is_root || !a.overlap) e.keep |= 1u;
    if (p.is_root && a.overlap) {  // C1 turnaround: final straight into the children
      for (int s = 0; s < p.nchild; ++s) {
        e.dst[1 + s] = p.child_buf[s];
        if (p.child_interior[s]) e.keep |= 2u << s;  // re-read by the child's DOWN
      }
      e.nout += p.nchild;
    }
  } else {
    e.nin = 1;
    e.src[0] = p.buf;
    for (int s = 0; s < p.nchild; ++s) {
      e.dst[s] = p.child_buf[s];
      if (p.child_interior[s]) e.keep |= 1u << s;
    }
    e.nout = p.nchild;
  }
  if (!a.l2_hints) e.keep = 0;
  return e;
}

// ---- L2 eviction priorities -------------------------------------------------------
// Every source is read for the last time (inputs once, partials once), so loads are
// evict_first; a store is evict_last when a later task of this launch re-reads it
// (partials, interior children's buffers), else evict_first (leaves' results).  With
// CCUBE_L2_HINTS=0 both policies are evict_normal.
struct L2Pol {
  uint64_t first, last;
};
__device__ __forceinline__ L2Pol make_pol(int on) {
  L2Pol p;
  if (on) {
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p.first));
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p.last));
  } else {
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p.first));
    p.last = p.first;
  }
  return p;
}
__device__ __forceinline__ uint4 ld_hint(const char *ptr, uint64_t pol) {
  uint4 v;
  asm volatile("ld.global.cg.L2::cache_hint.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(ptr), "l"(pol));
  return v;
}
__device__ __forceinline__ void st_hint(char *ptr, const uint4 &v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(ptr),
               "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol)
               : "memory");
}

// TMA datapath (kDatapathTma): a shared-memory ring of stages, each holding one block
// (<= kTmaSeg bytes) of every source; see tma_produce / tma_consume below.
constexpr uint32_t kTmaRing = 96u * 1024u;  // two CTAs per SM: 2 x 96 KB of the 228 KB
constexpr uint32_t kTmaSeg = 8192;          // bytes per source per stage (at most)
constexpr int kTmaMaxStages = 12;           // one source: 12 x 8 KB
constexpr uint32_t kTmaAbort = 0xffffffffu;

struct TmaDesc {
  uint64_t off;    // byte offset of the block in the buffers
  uint32_t len;    // bytes (kTmaAbort = stop)
  uint32_t kdone;  // after this block every chunk < kdone is finished (tree-local)
};

struct Shared {
  uint64_t ready;                // chunks whose inputs are available (control -> data)
  uint64_t done[kMaxDataWarps];  // chunks finished by data warp w (data -> control)
  int abort;
  uint64_t full[kTmaMaxStages];  // TMA: stage loaded (complete_tx)
  uint64_t empty[kTmaMaxStages]; // TMA: stage consumed by every consumer warp
  TmaDesc desc[kTmaMaxStages];
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

// ---- control / producer warp -------------------------------------------------------
// Releases chunks [pub, d) downstream: one fence, then one store per counter.
template <bool SYS>
__device__ __forceinline__ void publish(const LaunchArgs &a, const TreeParams &p, int role, int t,
                                        int j, uint32_t pub, uint32_t d, uint64_t base) {
  const int stride = j * kFlagStrideU64;
  const uint64_t v = base + d;
  fence_release<SYS>();
  if (does_sgd(a, p, role)) st_relaxed<SYS>(p.upd + stride, v);  // my weights updated
  if (role == kRoleUpdate) return;
  if (role == kRoleUp && !p.is_root) {
    st_relaxed<SYS>(p.head_out + stride, v);
    if (a.trace_up) trace_landing(a, p.self_local, t, pub, d, j, a.trace_up);
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

// A split task's release of chunks [pub, d): as publish(), but several writers (the
// two halves) may store each counter, so every store is a monotone max with release
// semantics (`red.release.max`): a half that publishes an older minimum can never move
// a counter back.
template <bool SYS>
__device__ __forceinline__ void red_max_release(uint64_t *p, uint64_t v) {
  if (SYS)
    asm volatile("red.release.sys.global.max.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else
    asm volatile("red.release.gpu.global.max.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
template <bool SYS>
__device__ __forceinline__ void fence_sc() {
  if (SYS)
    asm volatile("fence.sc.sys;" ::: "memory");
  else
    asm volatile("fence.sc.gpu;" ::: "memory");
}

template <bool SYS>
__device__ __forceinline__ void publish_max(const LaunchArgs &a, const TreeParams &p, int role,
                                            int t, int j, uint32_t pub, uint32_t d,
                                            uint64_t base) {
  const int stride = j * kFlagStrideU64;
  const uint64_t v = base + d;
  if (role == kRoleUp && !p.is_root) {
    red_max_release<SYS>(p.head_out + stride, v);
    if (a.trace_up) trace_landing(a, p.self_local, t, pub, d, j, a.trace_up);
    return;
  }
  if (role == kRoleUp) {  // root: the chunk is final in my own buffer
    red_max_release<SYS>(p.enq + stride, v);
    trace_landing(a, p.self_local, t, pub, d, j);
    if (!a.overlap) return;
  }
  for (int s = 0; s < p.nchild; ++s) {
    red_max_release<SYS>(p.child_enq[s] + stride, v);
    trace_landing(a, p.child_local[s], t, pub, d, j);
  }
}

// Half h of a split task has finished chunks < d (its own warps).  It records that
// in its progress slot, reads the other half's, and releases downstream the minimum
// of the two if that advanced.  The store-then-load on two slots is separated by a
// sequentially consistent fence in both halves, so of two halves finishing the same
// chunk at least one sees the other's progress: the minimum always gets published.
template <bool SYS>
__device__ __forceinline__ uint32_t publish_half(const LaunchArgs &a, const TreeParams &p,
                                                 int role, int t, int j, int half, uint32_t d,
                                                 uint32_t published, uint64_t base) {
  const int stride = j * kFlagStrideU64;
  fence_release<SYS>();                                 // my warps' stores, then my slot
  st_relaxed<SYS>(p.half_slot[half] + stride, base + d);
  fence_sc<SYS>();
  const uint64_t o = ld_acquire<SYS>(p.half_slot[half ^ 1] + stride);
  uint32_t m = o > base ? static_cast<uint32_t>(o - base < d ? o - base : d) : 0;
  if (m > published) {
    publish_max<SYS>(a, p, role, t, j, published, m, base);
    return m;
  }
  return published;
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

// Leaves on PULL edges: their inputs already sit where the parents read them.  One
// CTA per rank (the leaf group, task entries [first, first + n) after the grid)
// serves every tree in which the rank is a pulled leaf: its first warp publishes
// every such leaf's head on every channel at once, then waits until the rank's
// results have landed (the kernel completes only then).  All heads go out before
// any wait: a leaf's result in one tree may need its input in another.
template <bool SYS>
__device__ void pulled_leaves(const LaunchArgs &a, int first, int n) {
  const int lane = threadIdx.x & 31;
  const int J = static_cast<int>(a.nchannels);
  fence_release<SYS>();
  for (int x = lane; x < n * J; x += 32) {
    const Task &l = a.tasks[first + x / J];
    const TreeParams &p = a.params[l.local_rank * a.ntrees + l.tree];
    st_relaxed<SYS>(p.head_out + (x % J) * kFlagStrideU64, a.base[l.tree] + a.K[l.tree]);
  }
  for (int x = lane; x < n * J; x += 32) {
    const Task &l = a.tasks[first + x / J];
    const TreeParams &p = a.params[l.local_rank * a.ntrees + l.tree];
    const uint64_t target = a.base[l.tree] + a.K[l.tree];
    uint64_t *enq = p.enq + (x % J) * kFlagStrideU64;
    Watch wd;
    watch_reset(wd);
    while (ld_acquire<SYS>(enq) < target) {
      if (!watch_tick(wd, a, target, 0)) {
        st_relaxed<SYS>(enq, ~0ull);
        break;
      }
    }
  }
}

// ---- data warps -------------------------------------------------------------------
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

// ---- control warp + register-staged data warps ------------------------------
// The control warp polls upstream and publishes "chunks ready" in shared memory;
// each data warp streams its blocks (BlockIter) and reports, through a per-warp
// "done" counter, the chunk of its next block; the control warp publishes the
// minimum over the warps downstream.
template <bool SYS>
__device__ void control_warp(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
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
        st_relaxed<SYS>(p.upd + stride, ~0ull);
      }
      return;
    }
  }
  leaf_wait<SYS>(a, p, role, t, j);
}

// Split control (a.split_control): the two duties of control_warp run on two warps,
// so neither waits for the other.  The poll warp's loop is one global acquire round
// trip; the publish warp's loop is a shared-memory read, so a finished chunk is
// released downstream after the fence alone instead of after up to one upstream
// poll as well (the per-hop latency, alpha, that sets the pipeline's fill and drain).
template <bool SYS>
__device__ void poll_warp(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                          Shared &sh) {
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
  uint64_t ready = (role == kRoleUp && p.nchild == 0) || a.debug_nodep ? K : 0;  // a leaf's input is ready
  if (lane == 0) st_release_cta(&sh.ready, ready);
  Watch wd;
  watch_reset(wd);
  while (ready < K) {
    uint64_t v = up ? ld_acquire<SYS>(up) : ~0ull;
    v = warp_min(v);
    uint64_t r = v > base ? v - base : 0;
    if (r > K) r = K;
    if (hold_all && r < K) r = 0;
    if (r > ready) {
      __syncwarp();  // every lane's acquire happens before lane 0's release below
      ready = r;
      if (lane == 0) st_release_cta(&sh.ready, ready);
      watch_reset(wd);
    } else {
      if (*reinterpret_cast<volatile int *>(&sh.abort)) return;
      if (!watch_tick(wd, a, base + ready + 1, 0)) {
        if (lane == 0) {
          *reinterpret_cast<volatile int *>(&sh.abort) = 1;
          st_relaxed<SYS>(p.enq + stride, ~0ull);  // release gradient-queue waiters
          st_relaxed<SYS>(p.upd + stride, ~0ull);
        }
        return;
      }
    }
  }
}

template <bool SYS>
__device__ void publish_warp(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                             int W, Shared &sh, int half, int halves) {
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const uint64_t base = a.base[t];
  const int stride = j * kFlagStrideU64;
  uint32_t pub = 0;        // chunks my own warps finished
  uint32_t published = 0;  // split task: chunks released downstream (lane 0's view)
  Watch wd;
  watch_reset(wd);
  while (pub < K) {
    uint64_t d = lane < W ? ld_acquire_cta(&sh.done[lane]) : ~0ull;
    d = warp_min(d);
    if (d > pub) {
      __syncwarp();
      if (lane == 0) {
        if (halves == 1)
          publish<SYS>(a, p, role, t, j, pub, static_cast<uint32_t>(d), base);
        else
          published = publish_half<SYS>(a, p, role, t, j, half, static_cast<uint32_t>(d),
                                        published, base);
      }
      pub = static_cast<uint32_t>(d);
      watch_reset(wd);
    } else {  // (a split task needs no retry: the half that is behind publishes)
      if (*reinterpret_cast<volatile int *>(&sh.abort)) return;
      if (!watch_tick(wd, a, base + pub + 1, base + pub)) {
        if (lane == 0) {
          *reinterpret_cast<volatile int *>(&sh.abort) = 1;
          st_relaxed<SYS>(p.enq + stride, ~0ull);
          st_relaxed<SYS>(p.upd + stride, ~0ull);
        }
        return;
      }
    }
  }
  leaf_wait<SYS>(a, p, role, t, j);
}

// One data warp's stream: blocks of 32*U vectors (512*U bytes), see BlockIter.
// Lane l handles vectors l + 32u, u < U, of a block: U loads per source in
// flight, then the fixed-order combine and 128-bit stores to every destination.
// SGD (f2, fp32 only): the block's final gradient r also updates my weights,
// w <- w - alpha * r, as two IEEE-rounded operations (no FMA contraction; the
// oracle's reading R18) — one extra load and store stream, no extra pass.
__device__ __forceinline__ float sgd1(float w, float g, float alpha) {
  return __fsub_rn(w, __fmul_rn(alpha, g));
}
__device__ __forceinline__ uint4 sgd4(const uint4 &w, const uint4 &g, float alpha) {
  return make_uint4(__float_as_uint(sgd1(__uint_as_float(w.x), __uint_as_float(g.x), alpha)),
                    __float_as_uint(sgd1(__uint_as_float(w.y), __uint_as_float(g.y), alpha)),
                    __float_as_uint(sgd1(__uint_as_float(w.z), __uint_as_float(g.z), alpha)),
                    __float_as_uint(sgd1(__uint_as_float(w.w), __uint_as_float(g.w), alpha)));
}

template <int DT, int NIN, int NOUT, int U, bool SGD, bool OWN_FIRST = false>
__device__ void lsu_stream(const LaunchArgs &a, const Endpoints &e, int t, int j, int w, int W,
                           Shared &sh, int iw, int iW) {
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  constexpr uint32_t kSeg = 512u * U;
  const int lane = threadIdx.x & 31;
  const Geo g = make_geo<ES>(a, t, j);
  uint64_t ready = 0;
  uint32_t done_reported = 0;
  const L2Pol pol = make_pol(a.l2_hints);
  const float alpha = a.sgd_alpha;
  uint64_t dpol[NOUT > 0 ? NOUT : 1];
#pragma unroll
  for (int q = 0; q < NOUT; ++q) dpol[q] = (e.keep >> q) & 1u ? pol.last : pol.first;
  BlockIter it = iter_begin<kSeg>(g, iw);  // iw / iW: this warp among the task's CTAs
  // "done" = the chunk of my next block: I have no block in the chunks before my first
  // one, so say so now — otherwise chunk 0 is released only once every warp (including
  // those whose first block lies in chunk 1 or 2) has finished its first block, i.e.
  // each hop of the pipeline's fill would wait for two more upstream chunks.
  if (CCUBE_DONE_INIT && it.k > 0) {
    if (lane == 0) st_release_cta(&sh.done[w], it.k);
    done_reported = it.k;
  }
  // A combine (UP with children) reads my own input first: it is in my buffer from
  // the start, so its loads go out before the wait for the children's partials and
  // only the partials' (L2) latency stays on the hop's critical path.  Enabled for
  // the 6-warp CTAs (U = 6, the P = 8 geometry), where it measured 1.3% faster; the
  // 8-warp CTAs of the many-channel P = 2 / 4 geometry measured 1.4% slower with it
  // (round 2 session 2).
  constexpr bool kOwnFirst = CCUBE_OWN_FIRST && OWN_FIRST && NIN >= 2 && !SGD;
  while (it.k < g.K) {
    const uint32_t k = it.k;
    const uint32_t b0 = it.s * kSeg;
    const uint64_t off = it.sl.off + b0;
    const uint32_t len = min(kSeg, it.sl.len - b0);
    const uint32_t nvec = len / 16;
    uint4 x[U][NIN];
    uint4 wv[SGD ? U : 1];
    if constexpr (kOwnFirst) {
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (lane + 32u * u < nvec) x[u][0] = ld_hint(e.src[0] + off + lane * 16 + 512u * u, pol.first);
    }
    if (k >= ready) {
      uint64_t r = 0;
      if (lane == 0) {  // upstream not there yet: back off so busy warps get the issue slots
        while ((r = ld_acquire_cta(&sh.ready)) <= k &&
               !*reinterpret_cast<volatile int *>(&sh.abort))
          if (a.backoff_ns > 0) __nanosleep(a.backoff_ns);
      }
      r = __shfl_sync(0xffffffffu, r, 0);
      if (r <= k) return;  // aborted
      ready = r;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (lane + 32u * u < nvec) {
#pragma unroll
        for (int q = kOwnFirst ? 1 : 0; q < NIN; ++q)
          x[u][q] = ld_hint(e.src[q] + off + lane * 16 + 512u * u, pol.first);
        if constexpr (SGD) wv[u] = ld_hint(e.w + off + lane * 16 + 512u * u, pol.first);
      }
    }
    it.s += iW;  // advance while the loads are in flight (the loop is latency bound)
    iter_settle<kSeg>(g, it);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (lane + 32u * u < nvec) {
        const uint4 r = Combine<DT>::template vec<NIN>(x[u]);
#pragma unroll
        for (int q = 0; q < NOUT; ++q)
          st_hint(e.dst[q] + off + lane * 16 + 512u * u, r, dpol[q]);
        if constexpr (SGD)
          st_hint(e.w + off + lane * 16 + 512u * u, sgd4(wv[u], r, alpha), pol.first);
      }
    }
    if (len & 15u) {  // ragged end of the buffer (< 16 bytes, last block only)
      const uint64_t o = off + (len & ~15u);
      if (NOUT > 0) combine_scalar<DT>(e.src, NIN, e.dst, NOUT, o, len & 15u);
      if constexpr (SGD) {
        __syncwarp();  // the final values written just above (same lanes) come first
        for (uint32_t x4 = lane; x4 < (len & 15u) / 4; x4 += 32) {
          float *wp = reinterpret_cast<float *>(e.w + o) + x4;
          *wp = sgd1(*wp, reinterpret_cast<const float *>(e.gfinal + o)[x4], alpha);
        }
      }
    }
    if (it.k > done_reported) {
      __syncwarp();  // every lane's stores precede the release
      if (lane == 0) st_release_cta(&sh.done[w], it.k);
      done_reported = it.k;
    }
  }
  if (done_reported < g.K) {
    __syncwarp();
    if (lane == 0) st_release_cta(&sh.done[w], g.K);
  }
}

template <int DT, int NIN, bool SGD, int MAXT>
__device__ __forceinline__ void lsu_nout(const LaunchArgs &a, const Endpoints &e, int t, int j,
                                         int w, int W, Shared &sh, int iw, int iW) {
  // block = 2 KB (copies and combines); build-time overrides for experiments
  constexpr int U = NIN == 1 ? (MAXT <= 256 ? CCUBE_U_COPY_S : CCUBE_U_COPY) : u_combine(MAXT);
  if constexpr (SGD && DT == kFloat32 && NIN <= 2) {
    if (e.sgd) {  // root UP (NIN 2), interior DOWN and leaf UPDATE (NIN 1); U = 4 (2 KB)
      switch (e.nout) {
        case 0: lsu_stream<DT, NIN, 0, 4, true>(a, e, t, j, w, W, sh, iw, iW); return;
        case 1: lsu_stream<DT, NIN, 1, 4, true>(a, e, t, j, w, W, sh, iw, iW); return;
        default: lsu_stream<DT, NIN, 2, 4, true>(a, e, t, j, w, W, sh, iw, iW); return;
      }
    }
  }
  switch (e.nout) {
    case 1: lsu_stream<DT, NIN, 1, U, false, (MAXT <= 256)>(a, e, t, j, w, W, sh, iw, iW); break;
    case 2: lsu_stream<DT, NIN, 2, U, false, (MAXT <= 256)>(a, e, t, j, w, W, sh, iw, iW); break;
    default: lsu_stream<DT, NIN, 3, U, false, (MAXT <= 256)>(a, e, t, j, w, W, sh, iw, iW); break;
  }
}

// ---- TMA datapath (kDatapathTma) ---------------------------------------------------
// Data warp 0 is a producer: one lane walks this channel's blocks in chunk order (the
// same BlockIter as the LSU path, with kTmaSeg blocks and W = 1), waits for the
// control warp's "ready", and streams each block of every source into a ring stage
// with cp.async.bulk (mbarrier complete_tx).  Data warps 1..W-1 consume every stage:
// the fixed-order combine from shared memory, 128-bit stores to the destinations,
// then an arrive on the stage's "empty" barrier.  All sources are local (own buffer,
// own receive planes, or a same-GPU child's buffer on a PULL edge), so the bulk
// loads never cross NVLink; stores still go out as generic 128-bit stores, so the
// release chain to the control warp is the LSU path's.  The ring holds up to
// kTmaRing bytes in flight per CTA without registers: what the DRAM-heavy tasks
// lack in the register-staged path (tools/membench2.cu).
__device__ __forceinline__ void mbar_init(uint64_t *m, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *m) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(m)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *m, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(m)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_load(void *smem, const void *gptr, uint32_t bytes,
                                          uint64_t *m, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1], %2, [%3], %4;" ::"r"(smem_u32(smem)),
      "l"(gptr), "r"(bytes), "r"(smem_u32(m)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ int tma_nsrc(const Endpoints &e) { return e.nin + (e.sgd ? 1 : 0); }
__device__ __forceinline__ int tma_stages(int nsrc) {
  const int s = static_cast<int>(kTmaRing / (nsrc * kTmaSeg));
  return s < kTmaMaxStages ? s : kTmaMaxStages;
}

__device__ void tma_produce(const LaunchArgs &a, const Endpoints &e, int t, int j, Shared &sh,
                            char *ring) {
  const int ES = a.elem_size;
  const Geo g = ES == 2 ? make_geo<2>(a, t, j) : make_geo<4>(a, t, j);
  const int nsrc = tma_nsrc(e);
  const int S = tma_stages(nsrc);
  const char *src[kMaxIn + 1];
  for (int q = 0; q < e.nin; ++q) src[q] = e.src[q];
  if (e.sgd) src[e.nin] = e.w;
  const L2Pol pol = make_pol(a.l2_hints);
  uint64_t ready = 0;
  uint32_t i = 0;
  BlockIter it = iter_begin<kTmaSeg>(g, 0);
  bool aborted = false;
  while (it.k < g.K || i == 0) {  // an empty walk still sends one "all done" stage
    const uint32_t k = it.k;
    if (k < g.K && k >= ready) {
      uint64_t r;
      while ((r = ld_acquire_cta(&sh.ready)) <= k && !*reinterpret_cast<volatile int *>(&sh.abort))
        __nanosleep(64);
      if (r <= k) {
        aborted = true;
        break;
      }
      ready = r;
      // the upstream data was acquired through the generic proxy; the bulk loads
      // below read it through the async proxy
      asm volatile("fence.proxy.async.global;" ::: "memory");
    }
    const int s = static_cast<int>(i % S);
    if (i >= static_cast<uint32_t>(S)) mbar_wait(&sh.empty[s], ((i / S) - 1) & 1);
    uint64_t off = 0;
    uint32_t len = 0;
    if (k < g.K) {
      const uint32_t b0 = it.s * kTmaSeg;
      off = it.sl.off + b0;
      len = min(kTmaSeg, it.sl.len - b0);
      it.s += 1;
      iter_settle<kTmaSeg>(g, it);
    }
    sh.desc[s].off = off;
    sh.desc[s].len = len;
    sh.desc[s].kdone = it.k;
    const uint32_t vlen = len & ~15u;
    if (vlen) {
      mbar_expect_tx(&sh.full[s], vlen * nsrc);
      for (int q = 0; q < nsrc; ++q)
        bulk_load(ring + (s * nsrc + q) * kTmaSeg, src[q] + off, vlen, &sh.full[s], pol.first);
    } else {
      mbar_arrive(&sh.full[s]);
    }
    ++i;
  }
  if (aborted) {  // wake every consumer with a stop stage
    const int s = static_cast<int>(i % S);
    if (i >= static_cast<uint32_t>(S)) mbar_wait(&sh.empty[s], ((i / S) - 1) & 1);
    sh.desc[s].len = kTmaAbort;
    mbar_arrive(&sh.full[s]);
  }
}

template <int DT, int NIN, int NOUT, bool SGD>
__device__ void tma_consume(const LaunchArgs &a, const Endpoints &e, int t, int w, int cw,
                            int CW, Shared &sh, const char *ring) {
  constexpr int NSRC = NIN + (SGD ? 1 : 0);
  const int lane = threadIdx.x & 31;
  const int S = tma_stages(NSRC);
  const uint32_t K = a.K[t];
  const L2Pol pol = make_pol(a.l2_hints);
  const float alpha = a.sgd_alpha;
  uint64_t dpol[NOUT > 0 ? NOUT : 1];
#pragma unroll
  for (int q = 0; q < NOUT; ++q) dpol[q] = (e.keep >> q) & 1u ? pol.last : pol.first;
  uint32_t done_reported = 0;
  for (uint32_t i = 0;; ++i) {
    const int s = static_cast<int>(i % S);
    mbar_wait(&sh.full[s], (i / S) & 1);
    const TmaDesc d = sh.desc[s];
    if (d.len == kTmaAbort) return;
    const uint32_t nvec = d.len / 16;
    const uint4 *st = reinterpret_cast<const uint4 *>(ring + s * NSRC * kTmaSeg);
    constexpr uint32_t kSegVec = kTmaSeg / 16;
#pragma unroll 2
    for (uint32_t v = cw * 32 + lane; v < nvec; v += CW * 32) {
      uint4 x[NIN];
#pragma unroll
      for (int q = 0; q < NIN; ++q) x[q] = st[q * kSegVec + v];
      const uint4 r = Combine<DT>::template vec<NIN>(x);
      const uint64_t o = d.off + 16ull * v;
#pragma unroll
      for (int q = 0; q < NOUT; ++q) st_hint(e.dst[q] + o, r, dpol[q]);
      if constexpr (SGD) st_hint(e.w + o, sgd4(st[NIN * kSegVec + v], r, alpha), pol.first);
    }
    if ((d.len & 15u) && cw == 0) {  // ragged end of the buffer (< 16 bytes)
      const uint64_t o = d.off + (d.len & ~15u);
      if (NOUT > 0) combine_scalar<DT>(e.src, NIN, e.dst, NOUT, o, d.len & 15u);
      if constexpr (SGD) {
        __syncwarp();
        for (uint32_t x4 = lane; x4 < (d.len & 15u) / 4; x4 += 32) {
          float *wp = reinterpret_cast<float *>(e.w + o) + x4;
          *wp = sgd1(*wp, reinterpret_cast<const float *>(e.gfinal + o)[x4], alpha);
        }
      }
    }
    __syncwarp();  // every lane is done with the stage and its stores precede the release
    if (lane == 0) {
      mbar_arrive(&sh.empty[s]);
      if (d.kdone > done_reported) st_release_cta(&sh.done[w], d.kdone);
    }
    done_reported = d.kdone > done_reported ? d.kdone : done_reported;
    if (done_reported >= K) return;
  }
}

template <int DT, int NIN, bool SGD>
__device__ __forceinline__ void tma_nout(const LaunchArgs &a, const Endpoints &e, int t, int w,
                                         int cw, int CW, Shared &sh, const char *ring) {
  if constexpr (SGD && DT == kFloat32 && NIN <= 2) {
    if (e.sgd) {
      switch (e.nout) {
        case 0: tma_consume<DT, NIN, 0, true>(a, e, t, w, cw, CW, sh, ring); return;
        case 1: tma_consume<DT, NIN, 1, true>(a, e, t, w, cw, CW, sh, ring); return;
        default: tma_consume<DT, NIN, 2, true>(a, e, t, w, cw, CW, sh, ring); return;
      }
    }
  }
  switch (e.nout) {
    case 1: tma_consume<DT, NIN, 1, false>(a, e, t, w, cw, CW, sh, ring); break;
    case 2: tma_consume<DT, NIN, 2, false>(a, e, t, w, cw, CW, sh, ring); break;
    default: tma_consume<DT, NIN, 3, false>(a, e, t, w, cw, CW, sh, ring); break;
  }
}

// Data warp w of W on the TMA datapath: w == 0 produces (lane 0), the others consume.
template <int DT, bool SGD>
__device__ void tma_data_warp(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                              int w, int W, Shared &sh, char *ring) {
  Endpoints e = endpoints(a, p, role);
  if (!SGD) e.sgd = false;
  const int lane = threadIdx.x & 31;
  if (e.nout == 0 && !e.sgd) {  // nothing to write (cannot happen for scheduled tasks)
    if (lane == 0) st_release_cta(&sh.done[w], a.K[t]);
    return;
  }
  if (w == 0) {  // the producer is not a writer: it never holds the minimum back
    if (lane == 0) {
      st_release_cta(&sh.done[0], a.K[t]);
      tma_produce(a, e, t, j, sh, ring);
    }
    return;
  }
  switch (e.nin) {
    case 1: tma_nout<DT, 1, SGD>(a, e, t, w, w - 1, W - 1, sh, ring); break;
    case 2: tma_nout<DT, 2, SGD>(a, e, t, w, w - 1, W - 1, sh, ring); break;
    default: tma_nout<DT, 3, SGD>(a, e, t, w, w - 1, W - 1, sh, ring); break;
  }
}

template <int DT, bool SGD, int MAXT>
__device__ void data_warp(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                          int w, int W, Shared &sh, int half, int halves) {
  const int iw = half * W + w, iW = halves * W;  // a split task's halves interleave blocks
  Endpoints e = endpoints(a, p, role);
  if (!SGD) e.sgd = false;
  if (e.nout == 0 && !e.sgd) {  // nothing to write (cannot happen for scheduled tasks)
    if ((threadIdx.x & 31) == 0) st_release_cta(&sh.done[w], a.K[t]);
    return;
  }
  switch (e.nin) {
    case 1: lsu_nout<DT, 1, SGD, MAXT>(a, e, t, j, w, W, sh, iw, iW); break;
    case 2: lsu_nout<DT, 2, SGD, MAXT>(a, e, t, j, w, W, sh, iw, iW); break;
    default: lsu_nout<DT, 3, SGD, MAXT>(a, e, t, j, w, W, sh, iw, iW); break;
  }
}

// SGD = the fp32 variant with the fused update (f2); the plain kernels do not carry
// its code (register pressure).
// MAXT = the CTA size bound: 288 (8 data warps) or 256 (7 data warps, which leaves
// ptxas 128 registers per thread at two CTAs per SM instead of 96).
template <int DT, bool SYS, bool SGD, int MAXT>
__global__ void __launch_bounds__(MAXT, kMinBlocksPerSm) tree_allreduce_kernel(const LaunchArgs a) {
  __shared__ Shared sh;
  extern __shared__ __align__(128) char tma_ring[];  // kTmaRing bytes on the TMA datapath
  const Task task = a.tasks[blockIdx.x];
  const TreeParams &p = a.params[task.local_rank * a.ntrees + task.tree];
  const int warp = threadIdx.x >> 5;
  if (task.channel == kAllChannels) {  // the leaf group
    if (warp == 0) pulled_leaves<SYS>(a, task.half, task.halves);
    return;
  }
  const int nctl = a.split_control ? 2 : 1;  // control warps ahead of the data warps
  const int W = (blockDim.x >> 5) - nctl;
  const bool tma = a.tma != 0;
  if (threadIdx.x == 0) {
    sh.ready = 0;
    sh.abort = 0;
    if (tma) {
      for (int s = 0; s < kTmaMaxStages; ++s) {
        mbar_init(&sh.full[s], 1);
        mbar_init(&sh.empty[s], W - 1);
      }
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
  }
  if (threadIdx.x < kMaxDataWarps) sh.done[threadIdx.x] = 0;
  __syncthreads();
  if (warp == 0) {
    if (a.split_control)
      poll_warp<SYS>(a, p, task.role, task.tree, task.channel, sh);
    else
      control_warp<SYS>(a, p, task.role, task.tree, task.channel, W, sh);
  } else if (warp < nctl) {
    publish_warp<SYS>(a, p, task.role, task.tree, task.channel, W, sh, task.half, task.halves);
  } else if (tma) {
    tma_data_warp<DT, SGD>(a, p, task.role, task.tree, task.channel, warp - nctl, W, sh, tma_ring);
  } else {
    data_warp<DT, SGD, MAXT>(a, p, task.role, task.tree, task.channel, warp - nctl, W, sh,
                             task.half, task.halves);
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

// ---- LL protocol: single-chunk messages (latency-bound regime) ------------------
// The whole message is one chunk of tree 0 (a3: K = 1), so the fold is the same
// fixed-order tree fold as the chunked path (R2/R3) and the result is bitwise the
// same.  What changes is the hand-off: instead of data stores, a fence and a
// counter per hop (three loaded memory round trips), every 8 bytes of payload carry
// the call's epoch and the consumer polls the data itself (eq 3's alpha term).
// Phase 1 (reduce-up): per line, own ⊕ child_lo ⊕ child_hi, LL-stored into the
// parent's up-lines; the root instead writes the final value to its buffer and
// LL-stores it into its children's down-lines at once (C1 turnaround).
// Phase 2 (broadcast-down, non-root): wait for the down-line, write the final value
// to the buffer (the gradient queue), forward it to the children.  The last CTA of a
// rank publishes its Enqueue Semaphore (a8) so ccube_gradq_wait works unchanged.
template <bool SYS>
__device__ __forceinline__ uint4 ll_load(const char *p) {
  uint4 v;
  if (SYS)
    asm volatile("ld.relaxed.sys.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  else
    asm volatile("ld.relaxed.gpu.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  return v;
}
template <bool SYS>
__device__ __forceinline__ void ll_store(char *p, uint32_t d0, uint32_t d1, uint32_t e) {
  if (SYS)
    asm volatile("st.relaxed.sys.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(d0), "r"(e),
                 "r"(d1), "r"(e) : "memory");
  else
    asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(d0), "r"(e),
                 "r"(d1), "r"(e) : "memory");
}

// Poll the LL lines l0, l0 + stride, ... (kLLBatch of them, those < lines) until each
// carries the epoch; the loads of the lines still missing are issued together.
constexpr int kLLBatch = 4;
template <bool SYS>
__device__ __forceinline__ bool ll_wait_batch(const char *base, uint64_t l0, uint64_t stride,
                                              uint64_t lines, uint32_t e, const LLArgs &a,
                                              uint64_t &t0, uint32_t (&d0)[kLLBatch],
                                              uint32_t (&d1)[kLLBatch]) {
  uint32_t missing = 0;
#pragma unroll
  for (int i = 0; i < kLLBatch; ++i)
    if (l0 + i * stride < lines) missing |= 1u << i;
  uint32_t spins = 0;
  while (missing) {
    uint4 v[kLLBatch];
#pragma unroll
    for (int i = 0; i < kLLBatch; ++i)
      if (missing & (1u << i)) v[i] = ll_load<SYS>(base + 16 * (l0 + i * stride));
#pragma unroll
    for (int i = 0; i < kLLBatch; ++i)
      if ((missing & (1u << i)) && v[i].y == e && v[i].w == e) {
        d0[i] = v[i].x;
        d1[i] = v[i].z;
        missing &= ~(1u << i);
      }
    if (missing && (++spins & 255) == 0) {
      const uint64_t now = globaltimer();
      if (t0 == 0) t0 = now;
      if (*reinterpret_cast<volatile int *>(a.err) != 0) return false;
      if (now - t0 > a.timeout_ns) {
        volatile int *err = reinterpret_cast<volatile int *>(a.err);
        err[1] = static_cast<int>(blockIdx.x);
        err[2] = static_cast<int>(e);
        err[3] = static_cast<int>(missing);
        __threadfence_system();
        err[0] = 4;  // 4 = LL watchdog
        __threadfence_system();
        return false;
      }
    }
  }
  return true;
}

// One node's combine on a word pair: own, then each child's partial in ascending
// rank, left to right (R2); bf16 accumulates both halves in fp32 and rounds once
// per node output (R3); a leaf's own bits are forwarded untouched.
template <int DT>
__device__ __forceinline__ uint32_t ll_combine(uint32_t own, uint32_t c0, uint32_t c1, int n) {
  if (n == 0) return own;
  if (DT == kInt32) {
    own += c0;
    if (n > 1) own += c1;
    return own;
  } else if (DT == kFloat32) {
    float f = __fadd_rn(__uint_as_float(own), __uint_as_float(c0));
    if (n > 1) f = __fadd_rn(f, __uint_as_float(c1));
    return __float_as_uint(f);
  } else {
    float lo = __fadd_rn(bf_lo(own), bf_lo(c0)), hi = __fadd_rn(bf_hi(own), bf_hi(c0));
    if (n > 1) {
      lo = __fadd_rn(lo, bf_lo(c1));
      hi = __fadd_rn(hi, bf_hi(c1));
    }
    return bf_pack(lo, hi);
  }
}

// Guarded access to payload word w (4 bytes) of a buffer of `nbytes` bytes: the
// last word of an odd-length bf16 buffer holds one element.
__device__ __forceinline__ uint32_t ll_get(const char *buf, uint64_t w, uint64_t nbytes) {
  const uint64_t o = 4 * w;
  if (o + 4 <= nbytes) return *reinterpret_cast<const uint32_t *>(buf + o);
  if (o + 2 <= nbytes) return *reinterpret_cast<const uint16_t *>(buf + o);
  return 0;
}
__device__ __forceinline__ void ll_put(char *buf, uint64_t w, uint64_t nbytes, uint32_t v) {
  const uint64_t o = 4 * w;
  if (o + 4 <= nbytes)
    *reinterpret_cast<uint32_t *>(buf + o) = v;
  else if (o + 2 <= nbytes)
    *reinterpret_cast<uint16_t *>(buf + o) = static_cast<uint16_t>(v);
}

template <int DT, bool SYS>
__global__ void __launch_bounds__(512) ll_kernel(const LLArgs a) {
  const int rank = blockIdx.x / a.ctas;
  const int part = blockIdx.x % a.ctas;
  const LLRank &me = a.r[rank];
  const uint64_t nbytes = a.count * (DT == kBFloat16 ? 2 : 4);
  const uint64_t lines = (nbytes + 7) / 8;  // 8 payload bytes per 16-byte line
  const uint64_t stride = static_cast<uint64_t>(a.ctas) * blockDim.x;
  const uint32_t e = a.epoch;
  uint64_t t0 = 0;
  bool ok = true;
  // Each thread takes kLLBatch lines (l0, l0 + stride, ...) at a time, so its loads
  // and polls of those lines are in flight together.
  // phase 1: reduce-up (and the root's turnaround)
  for (uint64_t l0 = static_cast<uint64_t>(part) * blockDim.x + threadIdx.x; l0 < lines && ok;
       l0 += stride * kLLBatch) {
    uint32_t w0[kLLBatch], w1[kLLBatch], c0[kMaxChildren][kLLBatch] = {}, c1[kMaxChildren][kLLBatch] = {};
#pragma unroll
    for (int i = 0; i < kLLBatch; ++i) {
      const uint64_t l = l0 + i * stride;
      w0[i] = l < lines ? ll_get(me.buf, 2 * l, nbytes) : 0;
      w1[i] = l < lines ? ll_get(me.buf, 2 * l + 1, nbytes) : 0;
    }
#pragma unroll
    for (int s = 0; s < kMaxChildren; ++s)
      if (s < me.nchild && ok)
        ok = ll_wait_batch<SYS>(me.up_in[s], l0, stride, lines, e, a, t0, c0[s], c1[s]);
    if (!ok) break;
#pragma unroll
    for (int i = 0; i < kLLBatch; ++i) {
      const uint64_t l = l0 + i * stride;
      if (l >= lines) break;
      const uint32_t r0 = ll_combine<DT>(w0[i], c0[0][i], c0[1][i], me.nchild);
      const uint32_t r1 = ll_combine<DT>(w1[i], c1[0][i], c1[1][i], me.nchild);
      if (me.up_out) {
        ll_store<SYS>(me.up_out + 16 * l, r0, r1, e);
      } else {  // root: final
        ll_put(me.buf, 2 * l, nbytes, r0);
        ll_put(me.buf, 2 * l + 1, nbytes, r1);
        for (int s = 0; s < me.nchild; ++s) ll_store<SYS>(me.down_out[s] + 16 * l, r0, r1, e);
      }
    }
  }
  // phase 2: broadcast-down
  if (me.up_out) {
    for (uint64_t l0 = static_cast<uint64_t>(part) * blockDim.x + threadIdx.x;
         l0 < lines && ok; l0 += stride * kLLBatch) {
      uint32_t w0[kLLBatch], w1[kLLBatch];
      ok = ll_wait_batch<SYS>(me.down_in, l0, stride, lines, e, a, t0, w0, w1);
      if (!ok) break;
#pragma unroll
      for (int i = 0; i < kLLBatch; ++i) {
        const uint64_t l = l0 + i * stride;
        if (l >= lines) break;
        ll_put(me.buf, 2 * l, nbytes, w0[i]);
        ll_put(me.buf, 2 * l + 1, nbytes, w1[i]);
        for (int s = 0; s < me.nchild; ++s)
          ll_store<SYS>(me.down_out[s] + 16 * l, w0[i], w1[i], e);
      }
    }
  }
  // the rank's last CTA to finish publishes the Enqueue Semaphore: every final word
  // of this rank is in its buffer (the gradient-queue gate's condition, a8/a9)
  __syncthreads();
  if (threadIdx.x == 0) {
    fence_release<SYS>();
    if (a.ctas == 1) {  // the only CTA of the rank: no count to take
      st_relaxed<SYS>(me.enq, ok ? a.enq_value : ~0ull);
      return;
    }
    const unsigned long long prev = atomicAdd(reinterpret_cast<unsigned long long *>(me.done), 1ull);
    if (prev + 1 == a.done_base + a.ctas) {
      fence_release<SYS>();
      st_relaxed<SYS>(me.enq, ok ? a.enq_value : ~0ull);
    }
  }
}

template <int DT>
int launch_ll_t(const LLArgs &a, bool sys_scope, int nlocal, int threads, cudaStream_t s) {
  if (sys_scope)
    ll_kernel<DT, true><<<nlocal * a.ctas, threads, 0, s>>>(a);
  else
    ll_kernel<DT, false><<<nlocal * a.ctas, threads, 0, s>>>(a);
  return static_cast<int>(cudaGetLastError());
}

// Device-side barrier over tree 0 (ccube_barrier): warp i serves local rank i.
// Lane s < nchild waits for child s's "arrive" >= epoch; then lane 0 tells the
// parent (release store into the parent's counter), waits for the parent's
// "release" and passes it on to the children.  Once the root has heard from
// every subtree, every rank has entered the barrier; once a rank sees "release",
// the root had.  Same single-writer monotone counters as the AllReduce.
struct BarrierArgs {
  BarrierRank r[kMaxRanks];
  uint64_t epoch;
  int *err;
  uint64_t timeout_ns;
};

template <bool SYS>
__global__ void barrier_kernel(const BarrierArgs b) {
  const int lane = threadIdx.x & 31;
  const BarrierRank &me = b.r[threadIdx.x >> 5];
  const uint64_t t0 = globaltimer();
  bool ok = true;
  auto wait_ge = [&](const uint64_t *p) {
    while (ok && ld_acquire<SYS>(p) < b.epoch) {
      if (*reinterpret_cast<volatile int *>(b.err) != 0 || globaltimer() - t0 > b.timeout_ns) {
        if (*reinterpret_cast<volatile int *>(b.err) == 0) {
          *reinterpret_cast<volatile int *>(b.err) = 3;  // 3 = barrier timeout
          __threadfence_system();
        }
        ok = false;
      }
    }
  };
  if (lane < me.nchild) wait_ge(me.arrive[lane]);
  __syncwarp();
  if (lane == 0) {
    if (me.parent_arrive) {
      fence_release<SYS>();
      st_relaxed<SYS>(me.parent_arrive, b.epoch);
      wait_ge(me.release);
    }
    fence_release<SYS>();
    for (int s = 0; s < me.nchild; ++s) st_relaxed<SYS>(me.child_release[s], b.epoch);
  }
}

// Peer-bandwidth probe (ccube_measure_peer_bandwidth): the data warps' copy pattern —
// U 128-bit loads per lane from local HBM, then 128-bit stores with an evict_first
// policy — into destination blockIdx.y (a peer's HBM, mapped with CUDA IPC).
struct PeerCopyArgs {
  const char *src;
  char *dst[kMaxRanks];
  uint64_t nvec;
};

__global__ void __launch_bounds__(256) peer_copy_kernel(const PeerCopyArgs c) {
  constexpr int U = 4;
  const L2Pol pol = make_pol(1);
  char *dst = c.dst[blockIdx.y];
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x * U;
  for (uint64_t i0 = static_cast<uint64_t>(blockIdx.x) * blockDim.x * U + threadIdx.x;
       i0 < c.nvec; i0 += stride) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t i = i0 + static_cast<uint64_t>(u) * blockDim.x;
      if (i < c.nvec) v[u] = ld_hint(c.src + 16 * i, pol.first);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t i = i0 + static_cast<uint64_t>(u) * blockDim.x;
      if (i < c.nvec) st_hint(dst + 16 * i, v[u], pol.first);
    }
  }
}

// The kernel instance for a CTA of `threads` threads: the smallest size bucket
// (192 / 224 / 256 / 320) that holds it.
template <int DT, bool SYS, bool SGD>
void (*kernel_for(int threads))(const LaunchArgs) {
  if (threads <= 192) return tree_allreduce_kernel<DT, SYS, SGD, 192>;
  if (threads <= 224) return tree_allreduce_kernel<DT, SYS, SGD, 224>;
  if (threads <= 256) return tree_allreduce_kernel<DT, SYS, SGD, 256>;
  return tree_allreduce_kernel<DT, SYS, SGD, kMaxThreads>;
}

template <int DT, bool SYS, bool SGD>
int launch_t(const LaunchArgs &a, int grid, int threads, cudaStream_t s) {
  const size_t smem = a.tma ? kTmaRing : 0;
  auto *fn = kernel_for<DT, SYS, SGD>(threads);
  if (smem) cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  fn<<<grid, threads, smem, s>>>(a);
  return static_cast<int>(cudaGetLastError());
}

template <int DT, bool SYS, bool SGD>
const void *kernel_ptr(int threads) {
  return reinterpret_cast<const void *>(kernel_for<DT, SYS, SGD>(threads));
}

}  // namespace

int launch_tree_allreduce(const LaunchArgs &args, int dtype, bool sys_scope, int grid,
                          int threads, void *stream) {
  const int nctl = args.split_control ? 2 : 1;
  if (threads > kMaxThreads || threads < 32 * (nctl + 1) || threads % 32 ||
      threads / 32 - nctl > kMaxDataWarps)
    return cudaErrorInvalidValue;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (args.sgd) {
    if (dtype != kFloat32) return cudaErrorInvalidValue;
    return sys_scope ? launch_t<kFloat32, true, true>(args, grid, threads, s)
                     : launch_t<kFloat32, false, true>(args, grid, threads, s);
  }
  switch (dtype) {
    case kInt32:
      return sys_scope ? launch_t<kInt32, true, false>(args, grid, threads, s)
                       : launch_t<kInt32, false, false>(args, grid, threads, s);
    case kFloat32:
      return sys_scope ? launch_t<kFloat32, true, false>(args, grid, threads, s)
                       : launch_t<kFloat32, false, false>(args, grid, threads, s);
    case kBFloat16:
      return sys_scope ? launch_t<kBFloat16, true, false>(args, grid, threads, s)
                       : launch_t<kBFloat16, false, false>(args, grid, threads, s);
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

int launch_ll(const LLArgs &args, int dtype, bool sys_scope, int nlocal, int threads,
              void *stream) {
  if (nlocal < 1 || nlocal > kMaxRanks || args.ctas < 1 || threads < 32 || threads > 512)
    return cudaErrorInvalidValue;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  switch (dtype) {
    case kInt32: return launch_ll_t<kInt32>(args, sys_scope, nlocal, threads, s);
    case kFloat32: return launch_ll_t<kFloat32>(args, sys_scope, nlocal, threads, s);
    case kBFloat16: return launch_ll_t<kBFloat16>(args, sys_scope, nlocal, threads, s);
    default: return cudaErrorInvalidValue;
  }
}

int launch_barrier(const BarrierRank *ranks, int n, uint64_t epoch, int *err,
                   uint64_t timeout_ns, bool sys_scope, void *stream) {
  if (n <= 0 || n > kMaxRanks) return cudaErrorInvalidValue;
  BarrierArgs b;
  for (int i = 0; i < n; ++i) b.r[i] = ranks[i];
  b.epoch = epoch;
  b.err = err;
  b.timeout_ns = timeout_ns;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (sys_scope)
    barrier_kernel<true><<<1, 32 * n, 0, s>>>(b);
  else
    barrier_kernel<false><<<1, 32 * n, 0, s>>>(b);
  return static_cast<int>(cudaGetLastError());
}

int launch_peer_copy(const char *src, char *const *dst, int ndst, size_t bytes, int grid,
                     void *stream) {
  if (ndst < 1 || ndst > kMaxRanks || bytes % 16) return cudaErrorInvalidValue;
  PeerCopyArgs c;
  c.src = src;
  for (int i = 0; i < ndst; ++i) c.dst[i] = dst[i];
  c.nvec = bytes / 16;
  const int gx = grid / ndst > 0 ? grid / ndst : 1;
  peer_copy_kernel<<<dim3(gx, ndst), 256, 0, static_cast<cudaStream_t>(stream)>>>(c);
  return static_cast<int>(cudaGetLastError());
}

int query_max_blocks_per_sm(int dtype, bool sys_scope, bool sgd, int threads, int tma,
                            int *blocks) {
  const void *fn = nullptr;
  if (sgd) {
    fn = sys_scope ? kernel_ptr<kFloat32, true, true>(threads) : kernel_ptr<kFloat32, false, true>(threads);
  } else {
    switch (dtype) {
      case kInt32:
        fn = sys_scope ? kernel_ptr<kInt32, true, false>(threads) : kernel_ptr<kInt32, false, false>(threads);
        break;
      case kFloat32:
        fn = sys_scope ? kernel_ptr<kFloat32, true, false>(threads) : kernel_ptr<kFloat32, false, false>(threads);
        break;
      default:
        fn = sys_scope ? kernel_ptr<kBFloat16, true, false>(threads)
                       : kernel_ptr<kBFloat16, false, false>(threads);
        break;
    }
  }
  const size_t smem = tma ? kTmaRing : 0;
  if (smem) {
    const int rc = static_cast<int>(
        cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    if (rc != cudaSuccess) return rc;
  }
  return static_cast<int>(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, fn, threads, smem));
}

}  // namespace ccube
