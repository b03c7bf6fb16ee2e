// membench2.cu — attainable HBM bandwidth of the tree kernel's stream shapes
// (NIN sources -> NOUT destinations) with three datapaths, no flags:
//   lsu   : register-staged 128-bit loads/stores, U vectors per lane in flight (the
//           tree kernel's current datapath);
//   lsupf : the same with the next block's loads issued before the current block's
//           stores (register double buffering);
//   tma   : one elected thread streams blocks into an S-stage shared-memory ring with
//           cp.async.bulk (mbarrier complete_tx); copies (NIN == 1) go back out with
//           bulk stores straight from shared memory, combines are summed by the warps
//           from shared memory and stored with 128-bit st.global.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o membench2 tools/membench2.cu
//   ./membench2   (one JSON line per configuration; gbs counts every byte read + written)
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <vector>

#define CK(x)                                                                          \
  do {                                                                                 \
    cudaError_t e_ = (x);                                                              \
    if (e_ != cudaSuccess) {                                                           \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      return 1;                                                                        \
    }                                                                                  \
  } while (0)

struct Bufs {
  const char *src[3];
  char *dst[3];
};

__device__ __forceinline__ uint4 add4(uint4 a, uint4 b) {
  return make_uint4(__float_as_uint(__fadd_rn(__uint_as_float(a.x), __uint_as_float(b.x))),
                    __float_as_uint(__fadd_rn(__uint_as_float(a.y), __uint_as_float(b.y))),
                    __float_as_uint(__fadd_rn(__uint_as_float(a.z), __uint_as_float(b.z))),
                    __float_as_uint(__fadd_rn(__uint_as_float(a.w), __uint_as_float(b.w))));
}

// ---- LSU ------------------------------------------------------------------------
template <int NIN, int NOUT, int U, bool PF>
__global__ void __launch_bounds__(288, 2) lsu_kernel(Bufs b, size_t bytes) {
  const int lane = threadIdx.x & 31;
  const size_t gw = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const size_t nw = (gridDim.x * (size_t)blockDim.x) >> 5;
  const size_t blk = 512ull * U;
  const size_t nblk = bytes / blk;
  if (!PF) {
    for (size_t G = gw; G < nblk; G += nw) {
      const size_t off = G * blk + lane * 16;
      uint4 x[U][NIN];
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < NIN; ++q)
          x[u][q] = __ldcs(reinterpret_cast<const uint4 *>(b.src[q] + off + 512 * u));
#pragma unroll
      for (int u = 0; u < U; ++u) {
        uint4 r = x[u][0];
#pragma unroll
        for (int q = 1; q < NIN; ++q) r = add4(r, x[u][q]);
#pragma unroll
        for (int q = 0; q < NOUT; ++q) __stcs(reinterpret_cast<uint4 *>(b.dst[q] + off + 512 * u), r);
      }
    }
  } else {
    size_t G = gw;
    uint4 x[U][NIN];
    if (G < nblk) {
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < NIN; ++q)
          x[u][q] = __ldcs(reinterpret_cast<const uint4 *>(b.src[q] + G * blk + lane * 16 + 512 * u));
    }
    while (G < nblk) {
      const size_t off = G * blk + lane * 16;
      uint4 r[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        r[u] = x[u][0];
#pragma unroll
        for (int q = 1; q < NIN; ++q) r[u] = add4(r[u], x[u][q]);
      }
      const size_t Gn = G + nw;
      if (Gn < nblk) {
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int q = 0; q < NIN; ++q)
            x[u][q] = __ldcs(reinterpret_cast<const uint4 *>(b.src[q] + Gn * blk + lane * 16 + 512 * u));
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < NOUT; ++q) __stcs(reinterpret_cast<uint4 *>(b.dst[q] + off + 512 * u), r[u]);
      G = Gn;
    }
  }
}

// ---- TMA ------------------------------------------------------------------------
__device__ __forceinline__ uint32_t sm32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *m, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sm32(m)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sm32(m)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *m) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sm32(m)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *m, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(sm32(m)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_load(void *smem, const void *g, uint32_t bytes, uint64_t *m) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          sm32(smem)),
      "l"(g), "r"(bytes), "r"(sm32(m))
      : "memory");
}
__device__ __forceinline__ void bulk_store(void *g, const void *smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(g), "r"(sm32(smem)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// Copy (NIN == 1): one thread per CTA moves blocks gmem -> smem -> NOUT x gmem.
template <int NOUT, int S, int BLK>
__global__ void tma_copy_kernel(Bufs b, size_t bytes) {
  extern __shared__ __align__(128) char ring[];
  __shared__ __align__(8) uint64_t full[S];
  if (threadIdx.x != 0) return;
  for (int s = 0; s < S; ++s) mbar_init(&full[s], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const size_t nblk = bytes / BLK;
  // this CTA's blocks: G = blockIdx.x + i * gridDim.x
  size_t nmine = nblk > blockIdx.x ? (nblk - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  auto gofs = [&](size_t i) { return (blockIdx.x + i * gridDim.x) * (size_t)BLK; };
  for (size_t i = 0; i < nmine && i < S; ++i) {
    mbar_expect_tx(&full[i], BLK);
    bulk_load(ring + i * BLK, b.src[0] + gofs(i), BLK, &full[i]);
  }
  for (size_t i = 0; i < nmine; ++i) {
    const int s = i % S;
    mbar_wait(&full[s], (i / S) & 1);
    for (int q = 0; q < NOUT; ++q) bulk_store(b.dst[q] + gofs(i), ring + s * BLK, BLK);
    bulk_commit();
    // refill the stage of block i-1 (its stores were committed one group ago)
    if (i >= 1 && i - 1 + S < nmine) {
      bulk_wait_read<1>();
      const int sp = (i - 1) % S;
      mbar_expect_tx(&full[sp], BLK);
      bulk_load(ring + sp * BLK, b.src[0] + gofs(i - 1 + S), BLK, &full[sp]);
    }
  }
  bulk_wait_all();
}

// Combine (NIN >= 2): thread 0 of warp 0 produces; warps 1..W consume from smem.
template <int NIN, int NOUT, int S, int BLK>
__global__ void __launch_bounds__(288, 2) tma_combine_kernel(Bufs b, size_t bytes) {
  extern __shared__ __align__(128) char ring[];  // S stages x NIN x BLK
  __shared__ __align__(8) uint64_t full[S], empty[S];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int W = (blockDim.x >> 5) - 1;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], W);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const size_t nblk = bytes / BLK;
  const size_t nmine = nblk > blockIdx.x ? (nblk - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  auto gofs = [&](size_t i) { return (blockIdx.x + i * gridDim.x) * (size_t)BLK; };
  if (warp == 0) {
    if (lane != 0) return;
    for (size_t i = 0; i < nmine; ++i) {
      const int s = i % S;
      if (i >= S) mbar_wait(&empty[s], ((i / S) - 1) & 1);
      mbar_expect_tx(&full[s], NIN * BLK);
      for (int q = 0; q < NIN; ++q)
        bulk_load(ring + (s * NIN + q) * BLK, b.src[q] + gofs(i), BLK, &full[s]);
    }
    return;
  }
  const int w = warp - 1;
  constexpr int kVec = BLK / 16;
  for (size_t i = 0; i < nmine; ++i) {
    const int s = i % S;
    mbar_wait(&full[s], (i / S) & 1);
    const size_t go = gofs(i);
    for (int v = w * 32 + lane; v < kVec; v += W * 32) {
      uint4 r = reinterpret_cast<const uint4 *>(ring + (s * NIN) * BLK)[v];
#pragma unroll
      for (int q = 1; q < NIN; ++q) r = add4(r, reinterpret_cast<const uint4 *>(ring + (s * NIN + q) * BLK)[v]);
#pragma unroll
      for (int q = 0; q < NOUT; ++q) __stcs(reinterpret_cast<uint4 *>(b.dst[q] + go) + v, r);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);
  }
}

template <typename F>
float timeit(F launch) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int i = 0; i < 3; ++i) launch();
  cudaDeviceSynchronize();
  float best = 1e30f;
  for (int i = 0; i < 10; ++i) {
    cudaEventRecord(e0);
    launch();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    best = ms < best ? ms : best;
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return best;
}

static size_t g_bytes;
static void report(const char *dp, int nin, int nout, const char *extra, float ms) {
  const double gbs = (double)g_bytes * (nin + nout) / (ms * 1e-3) / 1e9;
  printf("{\"datapath\": \"%s\", \"nin\": %d, \"nout\": %d, %s, \"ms\": %.4f, \"gbs\": %.1f}\n", dp, nin,
         nout, extra, ms, gbs);
  fflush(stdout);
}

template <int NIN, int NOUT, int U, bool PF>
void run_lsu(Bufs b, int grid, int threads) {
  float ms = timeit([&] { lsu_kernel<NIN, NOUT, U, PF><<<grid, threads>>>(b, g_bytes); });
  char ex[128];
  snprintf(ex, sizeof ex, "\"U\": %d, \"grid\": %d, \"threads\": %d", U, grid, threads);
  report(PF ? "lsupf" : "lsu", NIN, NOUT, ex, ms);
}

template <int NOUT, int S, int BLK>
void run_tma_copy(Bufs b, int grid) {
  const int smem = S * BLK;
  cudaFuncSetAttribute(tma_copy_kernel<NOUT, S, BLK>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  float ms = timeit([&] { tma_copy_kernel<NOUT, S, BLK><<<grid, 32, smem>>>(b, g_bytes); });
  cudaError_t e = cudaGetLastError();
  char ex[160];
  snprintf(ex, sizeof ex, "\"S\": %d, \"blk\": %d, \"grid\": %d, \"err\": \"%s\"", S, BLK, grid,
           cudaGetErrorString(e));
  report("tma", 1, NOUT, ex, ms);
}

template <int NIN, int NOUT, int S, int BLK>
void run_tma_combine(Bufs b, int grid, int threads) {
  const int smem = S * NIN * BLK;
  cudaFuncSetAttribute(tma_combine_kernel<NIN, NOUT, S, BLK>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       smem);
  float ms = timeit([&] { tma_combine_kernel<NIN, NOUT, S, BLK><<<grid, threads, smem>>>(b, g_bytes); });
  cudaError_t e = cudaGetLastError();
  char ex[160];
  snprintf(ex, sizeof ex, "\"S\": %d, \"blk\": %d, \"grid\": %d, \"threads\": %d, \"err\": \"%s\"", S, BLK,
           grid, threads, cudaGetErrorString(e));
  report("tma", NIN, NOUT, ex, ms);
}

int main() {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  g_bytes = 256ull << 20;  // per buffer; 6 buffers = 1.5 GB >> L2
  char *p[6];
  for (int i = 0; i < 6; ++i) {
    CK(cudaMalloc(&p[i], g_bytes));
    CK(cudaMemset(p[i], 0, g_bytes));
  }
  Bufs b;
  for (int i = 0; i < 3; ++i) {
    b.src[i] = p[i];
    b.dst[i] = p[3 + i];
  }
  const int g2 = 2 * sms;
  if (getenv("MB2_PARTIAL")) {
    // per-CTA throughput when only part of the machine streams (the tree kernel's heavy
    // stage: 82 of 291 CTAs carry 6 of the 8 DRAM read streams at P=8)
    for (int g : {41, 82, 164}) {
      run_lsu<3, 1, 4, false>(b, g, 288);
      run_lsu<3, 1, 2, true>(b, g, 288);
      run_tma_combine<3, 1, 4, 8192>(b, g, 288);
      run_tma_combine<3, 1, 6, 8192>(b, g, 288);
      run_tma_combine<3, 1, 4, 16384>(b, g, 288);
      run_lsu<1, 2, 8, false>(b, g, 288);
      run_tma_copy<2, 4, 16384>(b, g);
      run_tma_copy<2, 8, 16384>(b, g);
    }
    return 0;
  }
  // copies 1 -> 1, 1 -> 2
  run_lsu<1, 1, 8, false>(b, g2, 288);
  run_lsu<1, 1, 4, true>(b, g2, 288);
  run_lsu<1, 1, 8, true>(b, g2, 288);
  run_lsu<1, 2, 8, false>(b, g2, 288);
  run_lsu<1, 2, 4, true>(b, g2, 288);
  for (int g : {sms, 2 * sms, 4 * sms}) {
    run_tma_copy<1, 4, 16384>(b, g);
    run_tma_copy<1, 6, 16384>(b, g);
    run_tma_copy<1, 4, 32768>(b, g);
    run_tma_copy<2, 4, 16384>(b, g);
    run_tma_copy<2, 6, 16384>(b, g);
  }
  // combines 3 -> 1, 2 -> 2
  run_lsu<3, 1, 4, false>(b, g2, 288);
  run_lsu<3, 1, 2, true>(b, g2, 288);
  run_lsu<3, 1, 4, true>(b, g2, 288);
  run_lsu<2, 2, 4, false>(b, g2, 288);
  run_lsu<2, 2, 4, true>(b, g2, 288);
  run_tma_combine<3, 1, 4, 8192>(b, g2, 288);
  run_tma_combine<3, 1, 3, 8192>(b, g2, 288);
  run_tma_combine<3, 1, 4, 4096>(b, g2, 288);
  run_tma_combine<3, 1, 6, 4096>(b, g2, 288);
  run_tma_combine<2, 2, 4, 8192>(b, g2, 288);
  run_tma_combine<3, 1, 4, 8192>(b, sms, 288);
  run_tma_combine<3, 1, 8, 8192>(b, sms, 288);
  return 0;
}
