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

constexpr int kUnroll = 4;
constexpr int kMaxThreads = 544;  // 16 data warps + the control warp
constexpr int kMaxDataWarps = 16;

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

// CTA-scope release/acquire on shared memory (control <-> data warps)
__device__ __forceinline__ void st_release_cta(uint64_t *p, uint64_t v) {
  asm volatile("st.release.cta.shared.u64 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(p)),
               "l"(v)
               : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_cta(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.cta.shared.u64 %0, [%1];"
               : "=l"(v)
               : "r"((uint32_t)__cvta_generic_to_shared(p))
               : "memory");
  return v;
}

__device__ __forceinline__ uint64_t warp_min(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t w = __shfl_xor_sync(0xffffffffu, v, o);
    v = w < v ? w : v;
  }
  return v;
}

struct Shared {
  uint64_t ready;                 // chunks whose inputs are available (control -> data)
  uint64_t done[kMaxDataWarps];   // chunks finished by data warp w (data -> control)
  int abort;
};

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

// One data warp's share of elements [elo, ehi): vectors w*32+lane, stepping W*32,
// U vectors per source in flight; the ragged scalar tail goes to warp 0.
// Sources are local HBM or (PULL) peer buffers; destinations may be peer memory.
template <int DT, int NIN, int NOUT>
__device__ __forceinline__ void process_warp(const char *const *src, char *const *dst,
                                             uint64_t elo, uint64_t ehi, int w, int W) {
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  constexpr int VE = 16 / ES;
  if (ehi <= elo) return;
  const uint64_t n = ehi - elo;
  const uint64_t nv = n / VE;
  const int lane = threadIdx.x & 31;
  const uint4 *s[NIN];
  uint4 *d[NOUT];
#pragma unroll
  for (int i = 0; i < NIN; ++i) s[i] = reinterpret_cast<const uint4 *>(src[i] + elo * ES);
#pragma unroll
  for (int i = 0; i < NOUT; ++i) d[i] = reinterpret_cast<uint4 *>(dst[i] + elo * ES);
  const uint64_t step = static_cast<uint64_t>(W) * 32;
  uint64_t i = static_cast<uint64_t>(w) * 32 + lane;
  for (; i + (kUnroll - 1) * step < nv; i += kUnroll * step) {
    uint4 v[kUnroll][NIN];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u)
#pragma unroll
      for (int q = 0; q < NIN; ++q) v[u][q] = __ldcg(s[q] + i + u * step);
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const uint4 r = Combine<DT>::template vec<NIN>(v[u]);
#pragma unroll
      for (int q = 0; q < NOUT; ++q) d[q][i + u * step] = r;
    }
  }
  for (; i < nv; i += step) {
    uint4 v[NIN];
#pragma unroll
    for (int q = 0; q < NIN; ++q) v[q] = __ldcg(s[q] + i);
    const uint4 r = Combine<DT>::template vec<NIN>(v);
#pragma unroll
    for (int q = 0; q < NOUT; ++q) d[q][i] = r;
  }
  if (w == 0) {
    const char *ss[NIN];
    char *dd[NOUT];
#pragma unroll
    for (int q = 0; q < NIN; ++q) ss[q] = src[q] + elo * ES;
#pragma unroll
    for (int q = 0; q < NOUT; ++q) dd[q] = dst[q] + elo * ES;
    for (uint64_t e = nv * VE + lane; e < n; e += 32)
      Combine<DT>::template scalar<NIN>(ss, dd, NOUT, e);
  }
}

template <int DT, int NIN>
__device__ __forceinline__ void process_nout(const char *const *src, char *const *dst, int nout,
                                             uint64_t elo, uint64_t ehi, int w, int W) {
  switch (nout) {
    case 1: process_warp<DT, NIN, 1>(src, dst, elo, ehi, w, W); break;
    case 2: process_warp<DT, NIN, 2>(src, dst, elo, ehi, w, W); break;
    case 3: process_warp<DT, NIN, 3>(src, dst, elo, ehi, w, W); break;
    default: break;
  }
}

template <int DT>
__device__ __forceinline__ void dispatch(const char *const *src, int nin, char *const *dst,
                                         int nout, uint64_t elo, uint64_t ehi, int w, int W) {
  switch (nin) {
    case 1: process_nout<DT, 1>(src, dst, nout, elo, ehi, w, W); break;
    case 2: process_nout<DT, 2>(src, dst, nout, elo, ehi, w, W); break;
    case 3: process_nout<DT, 3>(src, dst, nout, elo, ehi, w, W); break;
    default: break;
  }
}

__device__ __forceinline__ void slice_range(const LaunchArgs &a, int t, int j, uint32_t k,
                                            uint64_t *lo, uint64_t *hi) {
  const uint64_t c = static_cast<uint64_t>(k) * a.ntrees + t;  // R4: chunk c on tree c mod T
  const uint64_t cend = min((c + 1) * a.elems_per_chunk, a.count);
  const uint64_t l = c * a.elems_per_chunk + static_cast<uint64_t>(j) * a.slice_elems;
  const uint64_t h = min(l + a.slice_elems, cend);
  *lo = l;
  *hi = h > l ? h : l;
}

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

// ---- control warp --------------------------------------------------------------
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

template <bool SYS>
__device__ void control_warp(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                             int W, Shared &sh) {
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const uint64_t base = a.base[t];
  const int stride = j * kFlagStrideU64;
  // upstream counters: UP waits on each child's head, DOWN on my own semaphore
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
  // a leaf's kernel completes only once the whole result has landed in its buffer
  if (role == kRoleUp && !p.is_root && p.nchild == 0 && lane == 0) {
    watch_reset(wd);
    while (ld_acquire<SYS>(p.enq + stride) < base + K) {
      if (!watch_tick(wd, a, base + K, 0)) {
        st_relaxed<SYS>(p.enq + stride, ~0ull);
        return;
      }
    }
  }
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

// ---- data warps ----------------------------------------------------------------
template <int DT>
__device__ void data_warp(const LaunchArgs &a, const TreeParams &p, int role, int t, int j,
                          int w, int W, Shared &sh) {
  const int lane = threadIdx.x & 31;
  const uint32_t K = a.K[t];
  const char *src[3];
  char *dst[3];
  int nin, nout;
  if (role == kRoleUp) {
    nin = 1 + p.nchild;
    for (int q = 0; q < nin; ++q) src[q] = p.up_src[q];
    dst[0] = p.up_dst;
    nout = 1;
    if (p.is_root && a.overlap) {  // C1 turnaround: final straight into the children
      for (int s = 0; s < p.nchild; ++s) dst[1 + s] = p.child_buf[s];
      nout += p.nchild;
    }
  } else {
    nin = 1;
    src[0] = p.buf;
    for (int s = 0; s < p.nchild; ++s) dst[s] = p.child_buf[s];
    nout = p.nchild;
  }
  uint64_t ready = 0;
  for (uint32_t k = 0; k < K; ++k) {
    if (ready <= k) {
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
    uint64_t lo, hi;
    slice_range(a, t, j, k, &lo, &hi);
    dispatch<DT>(src, nin, dst, nout, lo, hi, w, W);
    __syncwarp();
    if (lane == 0) st_release_cta(&sh.done[w], k + 1);
  }
}

template <int DT, bool SYS>
__global__ void __launch_bounds__(kMaxThreads) tree_allreduce_kernel(const LaunchArgs a) {
  __shared__ Shared sh;
  const Task task = a.tasks[blockIdx.x];
  const TreeParams &p = a.params[task.local_rank * a.ntrees + task.tree];
  const int warp = threadIdx.x >> 5;
  if (task.channel == kAllChannels) {
    if (warp == 0) pulled_leaf<SYS>(a, p, task.tree);
    return;
  }
  const int W = (blockDim.x >> 5) - 1;
  if (threadIdx.x == 0) {
    sh.ready = 0;
    sh.abort = 0;
  }
  if (threadIdx.x < kMaxDataWarps) sh.done[threadIdx.x] = 0;
  __syncthreads();
  if (warp == 0)
    control_warp<SYS>(a, p, task.role, task.tree, task.channel, W, sh);
  else
    data_warp<DT>(a, p, task.role, task.tree, task.channel, warp - 1, W, sh);
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

template <int DT, bool SYS>
int launch_t(const LaunchArgs &a, int grid, int threads, cudaStream_t s) {
  tree_allreduce_kernel<DT, SYS><<<grid, threads, 0, s>>>(a);
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
      threads / 32 - 1 > kMaxDataWarps)
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

int query_max_blocks_per_sm(int dtype, bool sys_scope, int threads, int *blocks) {
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
  return static_cast<int>(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, fn, threads, 0));
}

}  // namespace ccube
