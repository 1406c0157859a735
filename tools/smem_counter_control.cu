// Control experiment for ncu's shared-memory bank-conflict counter (not product code).
//
// Question: does l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_{ld,st} count only
// addressing conflicts (several distinct 4-byte words in one bank within one 128-byte
// wavefront, Lemma 9.4's model), or also data-stage cycles lost to other
// traffic through the L1/SMEM data array (global loads returning into L1)?
//
// Every kernel here uses the textbook conflict-free pattern: in each 16-byte access,
// thread t of a warp touches bytes [16 t, 16 t + 16) of a 512-byte row, so each 8-lane
// phase covers all 32 banks exactly once (4 wavefronts per 512-byte request, the ideal).
// Any conflict the counter reports in these kernels is therefore not addressing.
//
//   mode 0  stream:    LDG.128 x8 -> STS.128 (linear) -> bar -> LDS.128 (linear, rotated
//                      by one warp: a real exchange) -> STG.128, 1+1 GiB, like config 3
//   mode 1  smem only: the same STS/LDS exchange repeated with no global traffic in the
//                      loop (one STG of a checksum per thread at the end)
//   mode 2  loads:     mode 0 with the global stores removed (LDG + exchange + checksum)
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o smem_ctl smem_counter_control.cu
// Run:   ./smem_ctl <mode> <iters> <vpt 8|16> <noalloc 0|1> <one tile per CTA 0|1>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int THREADS = 256;          // 8 warps
// VPT: 16-byte vectors per thread per tile (8: 32 KiB tiles as config 5-T's plan;
// 16: 64 KiB tiles and 16 loads in flight per thread as config 3's plan)

template <bool NOALLOC>
__device__ __forceinline__ int4 ldg(const int4* p) {
  int4 v;
  if (NOALLOC)   // the product kernels' coalesced-sigma load (ll_kernels.cuh ldg_v4<false>)
    asm volatile("ld.global.nc.L1::no_allocate.v4.b32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  else
    asm volatile("ld.global.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ void stg(int4* p, int4 v) {
  asm volatile("st.global.cs.v4.b32 [%0], {%1,%2,%3,%4};" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

template <int MODE, int VPT, bool NOALLOC>
__global__ void __launch_bounds__(THREADS) ctl_kernel(const int4* __restrict__ src, int4* __restrict__ dst,
                                                       long ntiles, int reps) {
  constexpr int TILE = THREADS * VPT;   // vectors per CTA tile
  extern __shared__ int4 buf[];
  const int t = threadIdx.x;
  const int w = t >> 5, l = t & 31;
  int4 acc = make_int4(0, 0, 0, 0);
  for (long tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    int4 r[VPT];
    const long base = tile * TILE;
#pragma unroll
    for (int k = 0; k < VPT; ++k) {
      if (MODE == 1) r[k] = make_int4(t + k, (int)tile, k, t);
      else r[k] = ldg<NOALLOC>(src + base + k * THREADS + t);     // coalesced 512 B per warp
    }
    for (int rep = 0; rep < (MODE == 1 ? reps : 1); ++rep) {
#pragma unroll
      for (int k = 0; k < VPT; ++k) buf[k * THREADS + t] = r[k];   // STS.128, lane-linear
      __syncthreads();
#pragma unroll
      for (int k = 0; k < VPT; ++k)                                // LDS.128, lane-linear,
        r[k] = buf[k * THREADS + (((w + 1) & 7) << 5) + l];       // next warp's row
      __syncthreads();
    }
#pragma unroll
    for (int k = 0; k < VPT; ++k) {
      if (MODE == 0) stg(dst + base + k * THREADS + t, r[k]);
      else { acc.x ^= r[k].x; acc.y ^= r[k].y; acc.z ^= r[k].z; acc.w ^= r[k].w; }
    }
  }
  if (MODE != 0) dst[(long)blockIdx.x * THREADS + t] = acc;
}

template <int VPT, bool NOALLOC>
static void run(int mode, int iters, int4* src, int4* dst, size_t bytes, int nsm, bool one_tile) {
  const long ntiles = long(bytes / (THREADS * VPT * sizeof(int4)));
  const int smem = THREADS * VPT * sizeof(int4);
  cudaFuncSetAttribute(ctl_kernel<0, VPT, NOALLOC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(ctl_kernel<1, VPT, NOALLOC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(ctl_kernel<2, VPT, NOALLOC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  // persistent grid (4 / 2 CTAs per SM) or one CTA per tile as the product's tile kernels
  const int grid = one_tile ? int(ntiles) : nsm * (VPT == 8 ? 4 : 2);
  auto launch = [&]() {
    if (mode == 0) ctl_kernel<0, VPT, NOALLOC><<<grid, THREADS, smem>>>(src, dst, ntiles, 1);
    else if (mode == 1) ctl_kernel<1, VPT, NOALLOC><<<grid, THREADS, smem>>>(src, dst, grid * 64L, 4);
    else ctl_kernel<2, VPT, NOALLOC><<<grid, THREADS, smem>>>(src, dst, ntiles, 1);
  };
  launch();
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  for (int i = 0; i < iters; ++i) launch();
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  ms /= iters;
  const double moved = mode == 0 ? 2.0 * bytes : mode == 2 ? double(bytes) : 0.0;
  printf("{\"mode\": %d, \"vpt\": %d, \"noalloc\": %d, \"one_tile_per_cta\": %d, \"ms\": %.4f, \"GBps\": %.1f, \"err\": \"%s\"}\n",
         mode, VPT, int(NOALLOC), int(one_tile), ms, moved / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
}

int main(int argc, char** argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 0;
  const int iters = argc > 2 ? atoi(argv[2]) : 10;
  const int vpt = argc > 3 ? atoi(argv[3]) : 8;
  const int noalloc = argc > 4 ? atoi(argv[4]) : 0;
  const bool one = argc > 5 && atoi(argv[5]) != 0;
  const size_t bytes = size_t(1) << 30;
  int4 *src, *dst;
  cudaMalloc(&src, bytes);
  cudaMalloc(&dst, bytes);
  cudaMemset(src, 1, bytes);
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  if (vpt == 16) { if (noalloc) run<16, true>(mode, iters, src, dst, bytes, nsm, one); else run<16, false>(mode, iters, src, dst, bytes, nsm, one); }
  else { if (noalloc) run<8, true>(mode, iters, src, dst, bytes, nsm, one); else run<8, false>(mode, iters, src, dst, bytes, nsm, one); }
  return 0;
}
