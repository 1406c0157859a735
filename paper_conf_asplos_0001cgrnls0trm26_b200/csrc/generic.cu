// Runtime-generic conversion kernel (compiled ahead of time for sm_100a).
//
// Used for maps the specialised tile kernels do not cover (broadcasting layouts,
// memory layouts whose pull map is not a bit permutation — Def 4.14 swizzles,
// P:240-276) and for exhaustive tiny-shape tests.  dst[y] = src[Q y] with Q given
// by its columns (XOR of the columns of the set bits of y): stores are
// coalesced (consecutive threads take consecutive y), loads are gathers.
#include <cuda_runtime.h>
#include <stdint.h>
#include <type_traits>

namespace ll {

struct QCols { unsigned long long col[64]; };

template <int W>
__global__ void __launch_bounds__(256) ll_generic_convert_kernel(const uint8_t* __restrict__ src,
                                                                 uint8_t* __restrict__ dst, QCols q, int nbits,
                                                                 unsigned long long nelem) {
  typedef typename std::conditional<W == 1, uint8_t,
          typename std::conditional<W == 2, uint16_t,
          typename std::conditional<W == 4, uint32_t, unsigned long long>::type>::type>::type T;
  const T* s = reinterpret_cast<const T*>(src);
  T* d = reinterpret_cast<T*>(dst);
  const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
  for (unsigned long long y = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; y < nelem; y += stride) {
    unsigned long long x = 0;
    for (int b = 0; b < nbits; ++b)
      if ((y >> b) & 1ull) x ^= q.col[b];
    d[y] = s[x];
  }
}

// NOOP plans (A = B, "equivalent layouts") with dst != src: the conversion is
// the identity on packed buffers, executed as a streaming copy in the tile kernels'
// shape — one 32 KiB tile per CTA (256 threads x 8 16-byte vectors, 512 contiguous
// bytes per warp instruction), all loads in flight before the stores, streaming cache
// hints, PDL like every other kernel.  Measured faster than cudaMemcpyAsync D2D on B200
// (profiles/r02_sweep_ceiling.jsonl).  A tail below 16 bytes (buffers < 16 bytes) is
// copied bytewise by CTA 0.
__global__ void __launch_bounds__(256) ll_copy_kernel(const uint4* __restrict__ src, uint4* __restrict__ dst,
                                                      unsigned long long nbytes) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  constexpr int V = 8;
  const unsigned long long nvec = nbytes >> 4;
  const unsigned long long base = (unsigned long long)blockIdx.x * (256ull * V) + threadIdx.x;
  uint4 r[V];
#pragma unroll
  for (int k = 0; k < V; ++k) {
    const unsigned long long i = base + 256ull * k;
    if (i < nvec)
      asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(r[k].x), "=r"(r[k].y), "=r"(r[k].z), "=r"(r[k].w) : "l"(src + i));
  }
#pragma unroll
  for (int k = 0; k < V; ++k) {
    const unsigned long long i = base + 256ull * k;
    if (i < nvec)
      asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(dst + i), "r"(r[k].x), "r"(r[k].y), "r"(r[k].z),
                   "r"(r[k].w) : "memory");
  }
  const unsigned tail = unsigned(nbytes & 15);
  if (tail && blockIdx.x == 0 && threadIdx.x < tail)
    reinterpret_cast<uint8_t*>(dst)[(nvec << 4) + threadIdx.x] = reinterpret_cast<const uint8_t*>(src)[(nvec << 4) + threadIdx.x];
}

void* copy_kernel_fn() { return reinterpret_cast<void*>(&ll_copy_kernel); }
unsigned copy_kernel_grid(unsigned long long nbytes) {
  const unsigned long long tiles = ((nbytes >> 4) + 2047) / 2048;
  return unsigned(tiles ? tiles : 1);
}

int launch_generic(const void* src, void* dst, const unsigned long long* cols, int nbits, unsigned long long nelem,
                   int w, cudaStream_t stream, int sms) {
  QCols q;
  for (int i = 0; i < 64; ++i) q.col[i] = i < nbits ? cols[i] : 0;
  unsigned long long blocks = (nelem + 255) / 256;
  unsigned long long cap = (unsigned long long)(sms > 0 ? sms : 148) * 16;
  unsigned grid = unsigned(blocks < cap ? blocks : cap);
  if (grid == 0) grid = 1;
  const uint8_t* s = static_cast<const uint8_t*>(src);
  uint8_t* d = static_cast<uint8_t*>(dst);
  switch (w) {
    case 1: ll_generic_convert_kernel<1><<<grid, 256, 0, stream>>>(s, d, q, nbits, nelem); break;
    case 2: ll_generic_convert_kernel<2><<<grid, 256, 0, stream>>>(s, d, q, nbits, nelem); break;
    case 4: ll_generic_convert_kernel<4><<<grid, 256, 0, stream>>>(s, d, q, nbits, nelem); break;
    default: ll_generic_convert_kernel<8><<<grid, 256, 0, stream>>>(s, d, q, nbits, nelem); break;
  }
  return int(cudaGetLastError());
}

// Flag barrier of the peer exchange (§8(f) N4).  flags[q] is rank q's flag buffer as
// mapped here; slot s of it holds the last epoch rank s announced to q.  Thread q
// announces `epoch` to rank q (release, system scope: the preceding kernel's peer
// stores are ordered before it) and waits until rank q announced it here (acquire).
// Epochs grow by one per barrier on every rank, so a peer can be at most one epoch
// ahead.  A rank that never arrives traps the kernel after 30 s (no GPU hang).
struct PeerFlags { unsigned* f[64]; };

__global__ void ll_peer_barrier_kernel(PeerFlags flags, int nranks, int rank, unsigned epoch) {
  const int q = threadIdx.x;
  if (q < nranks) {
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flags.f[q] + rank), "r"(epoch) : "memory");
    const unsigned* mine = flags.f[rank] + q;
    unsigned long long t0, t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    while (true) {
      unsigned v;
      asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(mine) : "memory");
      if (int(v - epoch) >= 0) break;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      if (t - t0 > 30000000000ull) __trap();
      __nanosleep(256);
    }
  }
  __syncthreads();
}

int launch_peer_barrier(void* const* flags, int nranks, int rank, unsigned epoch, cudaStream_t st) {
  PeerFlags f;
  for (int i = 0; i < 64; ++i) f.f[i] = i < nranks ? static_cast<unsigned*>(flags[i]) : nullptr;
  ll_peer_barrier_kernel<<<1, 64, 0, st>>>(f, nranks, rank, epoch);
  return int(cudaGetLastError());
}

}  // namespace ll
