// membench3.cu — register-staged streaming variants against the HBM copy peak (round 2):
//   lsu128 : the tree kernel's data-warp datapath (128-bit vectors, U per lane per
//            source, 2 CTAs/SM of 8 warps = 16 warps/SM);
//   lsu256 : the same with 256-bit vectors (ld/st.global.v8.u32, sm_100a);
//   occ128 : the same loop at full occupancy (8 CTAs of 8 warps per SM);
// for the stream shapes of the tree tasks: copy 1->1 / 1->2 (DOWN), 2->2 (C1 root),
// 3->1 (interior UP); and fold8, the loopback AllReduce's algorithmic floor done in
// one dependency-free pass (8 inputs read once, their fixed-order sum written to 8
// outputs) — the practical ceiling for any loopback AllReduce of that size.  gbs
// counts every byte read + written (best of 5 launches).  Argument: MiB per buffer.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o membench3 tools/membench3.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#define CK(x)                                                                          \
  do {                                                                                 \
    cudaError_t e_ = (x);                                                              \
    if (e_ != cudaSuccess) {                                                           \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      return 1;                                                                        \
    }                                                                                  \
  } while (0)

struct Bufs {
  const char *src[8];
  char *dst[8];
};

struct V8 {
  uint32_t w[8];
};

__device__ __forceinline__ float fa(uint32_t a, uint32_t b) {
  return __fadd_rn(__uint_as_float(a), __uint_as_float(b));
}

template <int VB>
struct Vec;
template <>
struct Vec<16> {
  using T = uint4;
  __device__ static T ld(const char *p) {
    T v;
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
  }
  __device__ static void st(char *p, const T &v) {
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
                 "r"(v.w) : "memory");
  }
  __device__ static T add(const T &a, const T &b) {
    return make_uint4(__float_as_uint(fa(a.x, b.x)), __float_as_uint(fa(a.y, b.y)),
                      __float_as_uint(fa(a.z, b.z)), __float_as_uint(fa(a.w, b.w)));
  }
};
template <>
struct Vec<32> {
  using T = V8;
  __device__ static T ld(const char *p) {
    T v;
    asm volatile("ld.global.cg.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v.w[0]), "=r"(v.w[1]), "=r"(v.w[2]), "=r"(v.w[3]), "=r"(v.w[4]),
                   "=r"(v.w[5]), "=r"(v.w[6]), "=r"(v.w[7])
                 : "l"(p));
    return v;
  }
  __device__ static void st(char *p, const T &v) {
    asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(v.w[0]),
                 "r"(v.w[1]), "r"(v.w[2]), "r"(v.w[3]), "r"(v.w[4]), "r"(v.w[5]), "r"(v.w[6]),
                 "r"(v.w[7])
                 : "memory");
  }
  __device__ static T add(const T &a, const T &b) {
    T r;
#pragma unroll
    for (int i = 0; i < 8; ++i) r.w[i] = __float_as_uint(fa(a.w[i], b.w[i]));
    return r;
  }
};

template <int NIN, int NOUT, int U, int VB>
__device__ __forceinline__ void stream(const Bufs &b, size_t bytes) {
  using V = Vec<VB>;
  const int lane = threadIdx.x & 31;
  const size_t gw = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const size_t nw = (gridDim.x * (size_t)blockDim.x) >> 5;
  const size_t blk = 32ull * VB * U;
  const size_t nblk = bytes / blk;
  for (size_t G = gw; G < nblk; G += nw) {
    const size_t off = G * blk + lane * VB;
    typename V::T x[U][NIN];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int q = 0; q < NIN; ++q) x[u][q] = V::ld(b.src[q] + off + 32 * VB * u);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      typename V::T r = x[u][0];
#pragma unroll
      for (int q = 1; q < NIN; ++q) r = V::add(r, x[u][q]);
#pragma unroll
      for (int q = 0; q < NOUT; ++q) V::st(b.dst[q] + off + 32 * VB * u, r);
    }
  }
}

template <int NIN, int NOUT, int U, int VB>
__global__ void __launch_bounds__(256, 2) k_tree(Bufs b, size_t bytes) {
  stream<NIN, NOUT, U, VB>(b, bytes);
}
template <int NIN, int NOUT, int U, int VB>
__global__ void __launch_bounds__(256, 8) k_occ(Bufs b, size_t bytes) {
  stream<NIN, NOUT, U, VB>(b, bytes);
}

// The loopback AllReduce's floor as one pass: every rank's input read once, the
// fixed-order sum computed in registers, every rank's output written once (2*P*N
// bytes, P = 8) — an upper bound for any loopback AllReduce of this size.
template <int U>
__global__ void __launch_bounds__(256, 2) k_fold8(Bufs b, size_t bytes) {
  const int lane = threadIdx.x & 31;
  const size_t gw = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const size_t nw = (gridDim.x * (size_t)blockDim.x) >> 5;
  const size_t blk = 512ull * U;
  for (size_t G = gw; G < bytes / blk; G += nw) {
    const size_t off = G * blk + lane * 16;
    uint4 x[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int q = 0; q < 8; ++q) x[u][q] = Vec<16>::ld(b.src[q] + off + 512 * u);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      uint4 r = x[u][0];
#pragma unroll
      for (int q = 1; q < 8; ++q) r = Vec<16>::add(r, x[u][q]);
#pragma unroll
      for (int q = 0; q < 8; ++q) Vec<16>::st(b.dst[q] + off + 512 * u, r);
    }
  }
}

size_t g_bytes;
int g_sms;

template <typename K>
int run(const char *name, K kern, int nin, int nout, int u, int vb, int grid, Bufs b) {
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  float best = 1e30f;
  for (int it = 0; it < 6; ++it) {
    CK(cudaEventRecord(e0));
    kern<<<grid, 256>>>(b, g_bytes);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    if (it > 0 && ms < best) best = ms;
  }
  const double gbs = (double)g_bytes * (nin + nout) / (best * 1e-3) / 1e9;
  printf("{\"variant\": \"%s\", \"nin\": %d, \"nout\": %d, \"U\": %d, \"vec_bytes\": %d, "
         "\"grid\": %d, \"bytes_per_buffer\": %zu, \"ms\": %.4f, \"gbs\": %.1f}\n",
         name, nin, nout, u, vb, grid, g_bytes, best, gbs);
  fflush(stdout);
  return 0;
}

#define RUN3(NIN, NOUT, U)                                                                \
  run("lsu128", k_tree<NIN, NOUT, U, 16>, NIN, NOUT, U, 16, 2 * g_sms, b);                \
  run("lsu256", k_tree<NIN, NOUT, (U > 1 ? U / 2 : 1), 32>, NIN, NOUT, (U > 1 ? U / 2 : 1), 32, \
      2 * g_sms, b);                                                                      \
  run("lsu256", k_tree<NIN, NOUT, U, 32>, NIN, NOUT, U, 32, 2 * g_sms, b);                \
  run("occ128", k_occ<NIN, NOUT, U, 16>, NIN, NOUT, U, 16, 8 * g_sms, b);

int main(int argc, char **argv) {
  CK(cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, 0));
  g_bytes = (argc > 1 ? (size_t)atol(argv[1]) : 256) << 20;
  char *p[16];
  for (int i = 0; i < 16; ++i) {
    CK(cudaMalloc(&p[i], g_bytes));
    CK(cudaMemset(p[i], 0, g_bytes));
  }
  Bufs b;
  for (int i = 0; i < 8; ++i) {
    b.src[i] = p[i];
    b.dst[i] = p[8 + i];
  }
  run("fold8", k_fold8<1>, 8, 8, 1, 16, 2 * g_sms, b);
  run("fold8", k_fold8<2>, 8, 8, 2, 16, 2 * g_sms, b);
  run("fold8", k_fold8<1>, 8, 8, 1, 16, 4 * g_sms, b);
  for (int i = 0; i < 3; ++i) b.dst[i] = p[3 + i];
  RUN3(1, 1, 4)
  RUN3(1, 1, 8)
  RUN3(1, 2, 4)
  RUN3(2, 2, 4)
  RUN3(3, 1, 4)
  run("lsu128", k_tree<1, 1, 4, 16>, 1, 1, 4, 16, 4 * g_sms, b);
  run("lsu128", k_tree<1, 2, 4, 16>, 1, 2, 4, 16, 4 * g_sms, b);
  return 0;
}
