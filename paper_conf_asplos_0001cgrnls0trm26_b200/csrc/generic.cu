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
