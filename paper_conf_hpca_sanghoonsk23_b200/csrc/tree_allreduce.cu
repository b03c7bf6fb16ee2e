// tree_allreduce.cu — the C-Cube hot path on sm_100a.
//
// One launch per AllReduce call ("one-shot").  Every CTA is one task
// (local rank, tree, role, channel): it owns slice `channel` of every chunk of
// `tree` and walks the tree-local chunks k = 0..K_t-1 in order (the tree keeps
// chunk order, Obs #3 P:L145; the gradient queue relies on it).
//
//   role UP   (a4, reduce-up): wait until each child's partial of chunk k
//             sits in my receive plane, combine own ⊕ child_lo ⊕ child_hi in that
//             fixed order (R2/R3) and push the result with 128-bit stores into the
//             parent's receive plane (NVLink peer memory), then release the
//             parent's head counter.  The root instead writes the final value into
//             its own buffer and — in C1 — straight into its children's
//             buffers, publishing their Enqueue Semaphores: the reduce->broadcast
//             turnaround costs no extra pass.
//   role DOWN (a5, broadcast-down): wait on my own Enqueue Semaphore (written by
//             my parent after it stored chunk k into my buffer, Fig 9), copy
//             chunk k from my buffer into each child's buffer and publish the
//             children's semaphores.  In B mode the root also runs a DOWN task that
//             starts only after all K_t chunks are reduced (Fig 7(a)).
// Leaves have no DOWN task; their UP task finally waits until the whole buffer
// has landed so that the kernel completes only when the result is final.
//
// Synchronisation (a7, replacing Fig 11's atomicCAS locks): single-writer
// monotone u64 counters; producer = CTA barrier + fence.acq_rel + relaxed store,
// consumer = one thread's acquire load + CTA barrier.  .sys scope when peers are
// other GPUs, .gpu scope in loopback.  Every spin has a %globaltimer watchdog.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace ccube {
namespace {

constexpr int kUnroll = 4;
constexpr int kMaxThreads = 512;

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

// Spin until *p >= target.  Returns false if the watchdog fired or another CTA
// already reported an error (then the caller must leave the kernel).
template <bool SYS>
__device__ bool wait_geq(const uint64_t *p, uint64_t target, int *err, uint64_t timeout_ns,
                         uint64_t *seen) {
  uint64_t v = ld_acquire<SYS>(p);
  if (v >= target) {
    *seen = v;
    return true;
  }
  const uint64_t t0 = globaltimer();
  uint64_t next_check = t0 + 1000000ull;  // look at the error word once per ms
  while (true) {
    v = ld_acquire<SYS>(p);
    if (v >= target) {
      *seen = v;
      return true;
    }
    const uint64_t now = globaltimer();
    if (now >= next_check) {
      if (*reinterpret_cast<volatile int *>(err) != 0) return false;
      if (now - t0 > timeout_ns) {
        reinterpret_cast<volatile int *>(err)[1] = static_cast<int>(blockIdx.x);
        reinterpret_cast<volatile int *>(err)[2] = static_cast<int>(target & 0x7fffffff);
        reinterpret_cast<volatile int *>(err)[3] = static_cast<int>(v & 0x7fffffff);
        __threadfence_system();
        *reinterpret_cast<volatile int *>(err) = 1;  // 1 = watchdog timeout
        __threadfence_system();
        return false;
      }
      next_check = now + 1000000ull;
    }
  }
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
  __device__ __forceinline__ static uint32_t word(const uint32_t *w, int n) {
    float lo = bf_lo(w[0]), hi = bf_hi(w[0]);
    for (int i = 1; i < n; ++i) {
      lo = __fadd_rn(lo, bf_lo(w[i]));
      hi = __fadd_rn(hi, bf_hi(w[i]));
    }
    return bf_round(lo) | (bf_round(hi) << 16);
  }
  template <int N>
  __device__ __forceinline__ static uint4 vec(const uint4 (&v)[N]) {
    if (N == 1) return v[0];  // a leaf forwards its own bits untouched
    uint32_t a[N], b[N], c[N], d[N];
#pragma unroll
    for (int i = 0; i < N; ++i) { a[i] = v[i].x; b[i] = v[i].y; c[i] = v[i].z; d[i] = v[i].w; }
    return make_uint4(word(a, N), word(b, N), word(c, N), word(d, N));
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

// Combine NIN sources element-wise over elements [elo, ehi) and store to NOUT
// destinations.  Sources are local HBM (own buffer / own receive planes);
// destinations may be peer memory.  128-bit accesses, kUnroll vectors in flight
// per thread per source, then the scalar tail of a ragged last chunk.
template <int DT, int NIN, int NOUT>
__device__ __forceinline__ void process(const char *const *src, char *const *dst, uint64_t elo,
                                        uint64_t ehi) {
  constexpr int ES = DT == kBFloat16 ? 2 : 4;
  constexpr int VE = 16 / ES;
  if (ehi <= elo) return;
  const uint64_t n = ehi - elo;
  const uint64_t nv = n / VE;
  const uint4 *s[NIN];
  uint4 *d[NOUT];
#pragma unroll
  for (int i = 0; i < NIN; ++i) s[i] = reinterpret_cast<const uint4 *>(src[i] + elo * ES);
#pragma unroll
  for (int i = 0; i < NOUT; ++i) d[i] = reinterpret_cast<uint4 *>(dst[i] + elo * ES);
  const uint64_t nt = blockDim.x;
  uint64_t i = threadIdx.x;
  for (; i + (kUnroll - 1) * nt < nv; i += kUnroll * nt) {
    uint4 v[kUnroll][NIN];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u)
#pragma unroll
      for (int q = 0; q < NIN; ++q) v[u][q] = __ldcg(s[q] + i + u * nt);
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const uint4 r = Combine<DT>::template vec<NIN>(v[u]);
#pragma unroll
      for (int q = 0; q < NOUT; ++q) d[q][i + u * nt] = r;
    }
  }
  for (; i < nv; i += nt) {
    uint4 v[NIN];
#pragma unroll
    for (int q = 0; q < NIN; ++q) v[q] = __ldcg(s[q] + i);
    const uint4 r = Combine<DT>::template vec<NIN>(v);
#pragma unroll
    for (int q = 0; q < NOUT; ++q) d[q][i] = r;
  }
  const char *ss[NIN];
  char *dd[NOUT];
#pragma unroll
  for (int q = 0; q < NIN; ++q) ss[q] = src[q] + elo * ES;
#pragma unroll
  for (int q = 0; q < NOUT; ++q) dd[q] = dst[q] + elo * ES;
  for (uint64_t e = nv * VE + threadIdx.x; e < n; e += nt)
    Combine<DT>::template scalar<NIN>(ss, dd, NOUT, e);
}

template <int DT, int NIN>
__device__ __forceinline__ void process_nout(const char *const *src, char *const *dst, int nout,
                                             uint64_t elo, uint64_t ehi) {
  switch (nout) {
    case 1: process<DT, NIN, 1>(src, dst, elo, ehi); break;
    case 2: process<DT, NIN, 2>(src, dst, elo, ehi); break;
    case 3: process<DT, NIN, 3>(src, dst, elo, ehi); break;
    default: break;
  }
}

template <int DT>
__device__ __forceinline__ void dispatch(const char *const *src, int nin, char *const *dst,
                                         int nout, uint64_t elo, uint64_t ehi) {
  switch (nin) {
    case 1: process_nout<DT, 1>(src, dst, nout, elo, ehi); break;
    case 2: process_nout<DT, 2>(src, dst, nout, elo, ehi); break;
    case 3: process_nout<DT, 3>(src, dst, nout, elo, ehi); break;
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

__device__ __forceinline__ void trace_landing(const LaunchArgs &a, int local, int t, uint32_t k,
                                              int j) {
  if (a.trace == nullptr || local < 0 || k >= a.trace_kmax) return;
  const uint64_t idx =
      ((static_cast<uint64_t>(local) * a.ntrees + t) * a.trace_kmax + k) * a.nchannels + j;
  a.trace[idx] = globaltimer();
}

template <int DT, bool SYS>
__device__ void up_role(const LaunchArgs &a, const TreeParams &p, int t, int j, int *sh_ok) {
  const uint32_t K = a.K[t];
  const uint64_t base = a.base[t];
  const int stride = j * kFlagStrideU64;
  uint64_t ready = 0;  // thread 0: tree-local chunks known complete at every child
  const char *src[3] = {p.buf, p.recv[0], p.recv[1]};
  char *dst[3];
  int nout = 1;
  if (p.is_root) {
    dst[0] = p.buf;
    if (a.overlap) {
      for (int s = 0; s < p.nchild; ++s) dst[1 + s] = p.child_buf[s];
      nout += p.nchild;
    }
  } else {
    dst[0] = p.parent_recv;
  }
  const int nin = 1 + p.nchild;
  for (uint32_t k = 0; k < K; ++k) {
    if (threadIdx.x == 0) {
      int ok = 1;
      if (p.nchild > 0 && ready <= k) {
        uint64_t m = ~0ull;
        for (int s = 0; s < p.nchild && ok; ++s) {
          uint64_t seen = 0;
          ok = wait_geq<SYS>(p.head_in[s] + stride, base + k + 1, a.err, a.timeout_ns, &seen);
          m = seen < m ? seen : m;
        }
        ready = m - base;
      }
      *sh_ok = ok;
    }
    __syncthreads();
    if (!*sh_ok) {
      if (threadIdx.x == 0) st_relaxed<SYS>(p.enq + stride, ~0ull);  // release gradq waiters
      return;
    }
    uint64_t lo, hi;
    slice_range(a, t, j, k, &lo, &hi);
    dispatch<DT>(src, nin, dst, nout, lo, hi);
    __syncthreads();  // every store of chunk k issued (and ordered) before the release
    if (threadIdx.x == 0) {
      const uint64_t v = base + k + 1;
      fence_release<SYS>();
      if (p.is_root) {
        st_relaxed<SYS>(p.enq + stride, v);
        trace_landing(a, p.self_local, t, k, j);
        if (a.overlap) {
          for (int s = 0; s < p.nchild; ++s) {
            st_relaxed<SYS>(p.child_enq[s] + stride, v);
            trace_landing(a, p.child_local[s], t, k, j);
          }
        }
      } else {
        st_relaxed<SYS>(p.head_out + stride, v);
      }
    }
  }
  if (!p.is_root && p.nchild == 0 && threadIdx.x == 0) {
    // leaf: the kernel may complete only once the whole result has landed here
    uint64_t seen;
    if (!wait_geq<SYS>(p.enq + stride, base + K, a.err, a.timeout_ns, &seen))
      st_relaxed<SYS>(p.enq + stride, ~0ull);
  }
}

template <int DT, bool SYS>
__device__ void down_role(const LaunchArgs &a, const TreeParams &p, int t, int j, int *sh_ok) {
  const uint32_t K = a.K[t];
  const uint64_t base = a.base[t];
  const int stride = j * kFlagStrideU64;
  uint64_t ready = 0;
  const char *src[1] = {p.buf};
  char *dst[2] = {p.child_buf[0], p.child_buf[1]};
  for (uint32_t k = 0; k < K; ++k) {
    if (threadIdx.x == 0) {
      int ok = 1;
      if (ready <= k) {
        // B mode root: hold every chunk until the whole reduction is done (Obs #1)
        const uint64_t target = p.is_root ? base + K : base + k + 1;
        uint64_t seen = 0;
        ok = wait_geq<SYS>(p.enq + stride, target, a.err, a.timeout_ns, &seen);
        ready = seen - base;
      }
      *sh_ok = ok;
    }
    __syncthreads();
    if (!*sh_ok) {
      if (threadIdx.x == 0) st_relaxed<SYS>(p.enq + stride, ~0ull);  // release gradq waiters
      return;
    }
    uint64_t lo, hi;
    slice_range(a, t, j, k, &lo, &hi);
    dispatch<DT>(src, 1, dst, p.nchild, lo, hi);
    __syncthreads();
    if (threadIdx.x == 0) {
      const uint64_t v = base + k + 1;
      fence_release<SYS>();
      for (int s = 0; s < p.nchild; ++s) {
        st_relaxed<SYS>(p.child_enq[s] + stride, v);
        trace_landing(a, p.child_local[s], t, k, j);
      }
    }
  }
}

template <int DT, bool SYS>
__global__ void __launch_bounds__(kMaxThreads) tree_allreduce_kernel(const LaunchArgs a) {
  __shared__ int sh_ok;
  const Task task = a.tasks[blockIdx.x];
  const TreeParams &p = a.params[task.local_rank * a.ntrees + task.tree];
  if (task.role == kRoleUp)
    up_role<DT, SYS>(a, p, task.tree, task.channel, &sh_ok);
  else
    down_role<DT, SYS>(a, p, task.tree, task.channel, &sh_ok);
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
    uint64_t seen;
    wait_geq<SYS>(g.ctr[i], g.target[i], g.err, g.timeout_ns, &seen);
  }
}

template <int DT, bool SYS>
int launch_t(const LaunchArgs &a, int grid, int threads, cudaStream_t s) {
  tree_allreduce_kernel<DT, SYS><<<grid, threads, 0, s>>>(a);
  return static_cast<int>(cudaGetLastError());
}

}  // namespace

int launch_tree_allreduce(const LaunchArgs &args, int dtype, bool sys_scope, int grid,
                          int threads, void *stream) {
  if (threads > kMaxThreads || threads < 32 || threads % 32) return cudaErrorInvalidValue;
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
      fn = sys_scope ? (const void *)tree_allreduce_kernel<kInt32, true>
                     : (const void *)tree_allreduce_kernel<kInt32, false>;
      break;
    case kFloat32:
      fn = sys_scope ? (const void *)tree_allreduce_kernel<kFloat32, true>
                     : (const void *)tree_allreduce_kernel<kFloat32, false>;
      break;
    default:
      fn = sys_scope ? (const void *)tree_allreduce_kernel<kBFloat16, true>
                     : (const void *)tree_allreduce_kernel<kBFloat16, false>;
      break;
  }
  return static_cast<int>(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, fn, threads, 0));
}

}  // namespace ccube
