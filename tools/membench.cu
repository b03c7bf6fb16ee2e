// membench.cu — attainable HBM bandwidth of the combine/copy shapes the tree kernel
// uses (NIN sources -> NOUT destinations, 128-bit accesses), as a function of CTAs
// per SM, warps per CTA and vectors in flight per lane.  No flags, no dependencies:
// this is the ceiling the tree kernel's data warps can reach.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o membench tools/membench.cu
//   ./membench            (prints one JSON line per configuration)
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <vector>

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e = (x);                                                       \
    if (e != cudaSuccess) {                                                    \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
      return 1;                                                                \
    }                                                                          \
  } while (0)

__device__ __forceinline__ uint4 add4(uint4 a, uint4 b) {
  return make_uint4(__float_as_uint(__uint_as_float(a.x) + __uint_as_float(b.x)),
                    __float_as_uint(__uint_as_float(a.y) + __uint_as_float(b.y)),
                    __float_as_uint(__uint_as_float(a.z) + __uint_as_float(b.z)),
                    __float_as_uint(__uint_as_float(a.w) + __uint_as_float(b.w)));
}

// Each warp streams blocks of 32*U vectors (G = gwarp, gwarp + nwarps, ...).
template <int NIN, int NOUT, int U, bool GLOBAL_ST, int REL = 0>
__global__ void stream_kernel(const char *const *src, char *const *dst, size_t bytes) {
  __shared__ unsigned long long done[32];
  const int lane = threadIdx.x & 31;
  const size_t gw = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const size_t nw = (gridDim.x * (size_t)blockDim.x) >> 5;
  const size_t blk = 512ull * U;
  const size_t nblk = bytes / blk;
  const char *s[NIN];
  char *d[NOUT];
#pragma unroll
  for (int q = 0; q < NIN; ++q) s[q] = src[q];
#pragma unroll
  for (int q = 0; q < NOUT; ++q) d[q] = dst[q];
  for (size_t G = gw; G < nblk; G += nw) {
    const size_t off = G * blk + lane * 16;
    uint4 x[U][NIN];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int q = 0; q < NIN; ++q)
        x[u][q] = __ldcg(reinterpret_cast<const uint4 *>(s[q] + off + 512 * u));
#pragma unroll
    for (int u = 0; u < U; ++u) {
      uint4 r = x[u][0];
#pragma unroll
      for (int q = 1; q < NIN; ++q) r = add4(r, x[u][q]);
#pragma unroll
      for (int q = 0; q < NOUT; ++q) {
        if (GLOBAL_ST)
          __stcg(reinterpret_cast<uint4 *>(d[q] + off + 512 * u), r);
        else
          *reinterpret_cast<uint4 *>(d[q] + off + 512 * u) = r;
      }
    }
    if (REL == 1) {
      __syncwarp();
      if (lane == 0)
        asm volatile("st.release.cta.shared.u64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(&done[threadIdx.x >> 5])), "l"((unsigned long long)G) : "memory");
    } else if (REL == 2) {
      __threadfence_block();
    } else if (REL == 3) {
      __syncwarp();
      if (lane == 0) *reinterpret_cast<volatile unsigned long long *>(&done[threadIdx.x >> 5]) = G;
    } else if (REL == 4) {
      __syncwarp();
      if (lane == 0) {
        asm volatile("fence.acq_rel.cta;" ::: "memory");
        *reinterpret_cast<volatile unsigned long long *>(&done[threadIdx.x >> 5]) = G;
      }
    }
  }
}

template <int NIN, int NOUT, int U, bool GS, int REL = 0>
int run(const char *name, char **bufs, char **d_src, char **d_dst, size_t bytes, int sms,
        int ctas_per_sm, int threads, float *ms_out) {
  (void)bufs;
  const int grid = sms * ctas_per_sm;
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  for (int i = 0; i < 3; ++i) stream_kernel<NIN, NOUT, U, GS, REL><<<grid, threads>>>(d_src, d_dst, bytes);
  CK(cudaDeviceSynchronize());
  std::vector<float> v;
  for (int i = 0; i < 10; ++i) {
    CK(cudaEventRecord(e0));
    stream_kernel<NIN, NOUT, U, GS, REL><<<grid, threads>>>(d_src, d_dst, bytes);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    v.push_back(ms);
  }
  float best = v[0];
  for (float x : v) best = x < best ? x : best;
  const double gbs = (double)bytes * (NIN + NOUT) / (best * 1e-3) / 1e9;
  printf("{\"shape\": \"%s\", \"nin\": %d, \"nout\": %d, \"U\": %d, \"global_st\": %d, "
         "\"rel\": %d, \"ctas_per_sm\": %d, \"threads\": %d, \"ms\": %.4f, \"gbs\": %.1f}\n",
         name, NIN, NOUT, U, (int)GS, REL, ctas_per_sm, threads, best, gbs);
  *ms_out = best;
  return 0;
}

int main() {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const size_t bytes = 256ull << 20;  // per buffer; 6 buffers = 1.5 GB >> L2
  char *b[6];
  for (int i = 0; i < 6; ++i) {
    CK(cudaMalloc(&b[i], bytes));
    CK(cudaMemset(b[i], 0, bytes));
  }
  char **d_src, **d_dst;
  CK(cudaMalloc(&d_src, 3 * sizeof(char *)));
  CK(cudaMalloc(&d_dst, 3 * sizeof(char *)));
  CK(cudaMemcpy(d_src, b, 3 * sizeof(char *), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_dst, b + 3, 3 * sizeof(char *), cudaMemcpyHostToDevice));
  float ms;
  for (int c : {1, 2}) {
    run<2, 2, 4, false, 0>("sum2to2", b, d_src, d_dst, bytes, sms, c, 256, &ms);
    run<2, 2, 4, false, 1>("sum2to2", b, d_src, d_dst, bytes, sms, c, 256, &ms);
    run<2, 2, 4, false, 2>("sum2to2", b, d_src, d_dst, bytes, sms, c, 256, &ms);
    run<2, 2, 4, false, 3>("sum2to2", b, d_src, d_dst, bytes, sms, c, 256, &ms);
    run<2, 2, 4, false, 4>("sum2to2", b, d_src, d_dst, bytes, sms, c, 256, &ms);
    run<3, 1, 4, false, 0>("sum3", b, d_src, d_dst, bytes, sms, c, 256, &ms);
    run<3, 1, 4, false, 1>("sum3", b, d_src, d_dst, bytes, sms, c, 256, &ms);
  }
  // 64 CTAs (P=2 loopback shape)
  for (int c : {0}) {
    (void)c;
    const int g64 = 64;
    run<2, 2, 4, false, 0>("sum2to2_g64", b, d_src, d_dst, bytes, g64, 1, 256, &ms);
    run<2, 2, 4, false, 1>("sum2to2_g64", b, d_src, d_dst, bytes, g64, 1, 256, &ms);
    run<2, 2, 4, false, 2>("sum2to2_g64", b, d_src, d_dst, bytes, g64, 1, 256, &ms);
    run<2, 2, 4, false, 3>("sum2to2_g64", b, d_src, d_dst, bytes, g64, 1, 256, &ms);
  }
  // partial-SM grids (the P=2 loopback case: 64 CTAs)
  for (int g : {16, 32, 64, 96, 128}) {
    const int grid = g;
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    for (int i = 0; i < 3; ++i) stream_kernel<2, 2, 4, false><<<grid, 256>>>(d_src, d_dst, bytes);
    CK(cudaEventRecord(e0));
    stream_kernel<2, 2, 4, false><<<grid, 256>>>(d_src, d_dst, bytes);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    CK(cudaEventElapsedTime(&ms, e0, e1));
    printf("{\"shape\": \"sum2to2\", \"grid\": %d, \"threads\": 256, \"ms\": %.4f, \"gbs\": %.1f, "
           "\"gbs_per_cta\": %.1f}\n",
           grid, ms, bytes * 4.0 / (ms * 1e-3) / 1e9, bytes * 4.0 / (ms * 1e-3) / 1e9 / grid);
  }
  return 0;
}
