// ll_kernels.cuh — sm_100a kernel templates for the linear-layout conversion hot path.
//
// Hand-written CUDA; specialised per plan by codegen.cpp, which emits a `struct P`
// of compile-time tables (plan constants) and instantiates the entry points at the
// end of this file.  Compiled with NVRTC for sm_100a (jit.cpp) and cached.
//
// Every register index below is a compile-time constant (static_for), so the
// per-thread register file is addressed statically: register permutations are
// free renamings, lane-dependent choices are selp networks (P:371-389 via the
// affine decomposition of DESIGN.md §5.2).
//
// Rows of SURVEY §8(a): a5 HBM load (ld_tile), a6 REGPERM, a7 SHUFFLE, a8 SMEM,
// a9 CTA (grid map), a10 HBM store (st_tile), a11 gather, a12 reduce.

typedef unsigned int u32;
typedef unsigned long long u64;
typedef unsigned short u16;
typedef unsigned char u8;

namespace std {
template <bool B, class T, class F> struct conditional { typedef T type; };
template <class T, class F> struct conditional<false, T, F> { typedef F type; };
}  // namespace std

// ------------------------------------------------------------------ compile-time loops
template <int V> struct IC { static constexpr int value = V; };
template <int I, int N, bool Small = (N - I <= 1)> struct SFor;
template <int I, int N> struct SFor<I, N, true> {
  template <class F> __device__ __forceinline__ static void run(F& f) {
    if constexpr (N - I == 1) f(IC<I>{});
  }
};
template <int I, int N> struct SFor<I, N, false> {
  template <class F> __device__ __forceinline__ static void run(F& f) {
    SFor<I, (I + N) / 2>::run(f);
    SFor<(I + N) / 2, N>::run(f);
  }
};
template <int N, class F> __device__ __forceinline__ void static_for(F&& f) { SFor<0, N>::run(f); }

// ------------------------------------------------------------------ element access
// Registers are 32-bit words; an element of W bytes (W in 1, 2, 4) at slot e lives
// in word e*W/4 at byte (e*W) % 4.
template <int W, int E> __device__ __forceinline__ u32 get_e(const u32* r) {
  if constexpr (W == 4) return r[E];
  else if constexpr (W == 2) return (r[E >> 1] >> (16 * (E & 1))) & 0xffffu;
  else return (r[E >> 2] >> (8 * (E & 3))) & 0xffu;
}
template <int W, int E> __device__ __forceinline__ void set_e(u32* r, u32 v) {
  if constexpr (W == 4) r[E] = v;
  else if constexpr (W == 2) {
    constexpr int s = 16 * (E & 1);
    r[E >> 1] = (r[E >> 1] & ~(0xffffu << s)) | (v << s);
  } else {
    constexpr int s = 8 * (E & 3);
    r[E >> 2] = (r[E >> 2] & ~(0xffu << s)) | (v << s);
  }
}

// ------------------------------------------------------------------ global memory
// Global loads.  L1A = false: streaming (.L1::no_allocate) for coalesced σ, where a
// warp instruction covers whole lines; L1A = true: L1-allocating read-only loads for
// per-thread-contiguous σ, where consecutive instructions of a lane share sectors.
template <bool L1A>
__device__ __forceinline__ void ldg_v4(const u8* p, u32& a, u32& b, u32& c, u32& d) {
  if constexpr (L1A)
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "l"(p));
}
template <bool L1A>
__device__ __forceinline__ void ldg_v2(const u8* p, u32& a, u32& b) {
  if constexpr (L1A)
    asm volatile("ld.global.nc.v2.u32 {%0,%1}, [%2];" : "=r"(a), "=r"(b) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0,%1}, [%2];" : "=r"(a), "=r"(b) : "l"(p));
}
template <bool L1A>
__device__ __forceinline__ u32 ldg_b32(const u8* p) {
  u32 a;
  if constexpr (L1A)
    asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(a) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(a) : "l"(p));
  return a;
}
// Global stores.  HINT 0: default (write-back); 1: .cs (streaming, evict-first).
template <int HINT>
__device__ __forceinline__ void stg_v4(u8* p, u32 a, u32 b, u32 c, u32 d) {
  if constexpr (HINT == 1)
    asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
  else
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}
template <int HINT>
__device__ __forceinline__ void stg_v2(u8* p, u32 a, u32 b) {
  if constexpr (HINT == 1)
    asm volatile("st.global.cs.v2.u32 [%0], {%1,%2};" ::"l"(p), "r"(a), "r"(b) : "memory");
  else
    asm volatile("st.global.v2.u32 [%0], {%1,%2};" ::"l"(p), "r"(a), "r"(b) : "memory");
}
template <int HINT>
__device__ __forceinline__ void stg_b32(u8* p, u32 a) {
  if constexpr (HINT == 1)
    asm volatile("st.global.cs.u32 [%0], %1;" ::"l"(p), "r"(a) : "memory");
  else
    asm volatile("st.global.u32 [%0], %1;" ::"l"(p), "r"(a) : "memory");
}

__device__ __forceinline__ void lds_v4(u32 addr, u32& a, u32& b, u32& c, u32& d) {
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "r"(addr) : "memory");
}
// cp.async (LDGSTS): 16 bytes global -> shared, bypassing L1 and registers; groups
// complete in order (cp.async.wait_group N: all but the newest N groups have landed).
__device__ __forceinline__ void cp_async16(u32 dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// Load vector K of the thread (2^VL elements of W bytes starting at slot K<<VL).
template <int W, int VL, int K, int NW, bool L1A = false>
__device__ __forceinline__ void load_vec(u32 (&r)[NW], const u8* p) {
  constexpr int VB = W << VL;                 // vector bytes
  constexpr int E0 = K << VL;
  if constexpr (VB == 16) {
    ldg_v4<L1A>(p, r[E0 * W / 4 + 0], r[E0 * W / 4 + 1], r[E0 * W / 4 + 2], r[E0 * W / 4 + 3]);
  } else if constexpr (VB == 8) {
    ldg_v2<L1A>(p, r[E0 * W / 4 + 0], r[E0 * W / 4 + 1]);
  } else if constexpr (VB == 4) {
    r[E0 * W / 4] = ldg_b32<L1A>(p);
  } else if constexpr (VB == 2) {
    set_e<2, E0 * W / 2>(r, u32(*reinterpret_cast<const u16*>(p)));
  } else {
    static_assert(VB == 1, "global vector width must be 1, 2, 4, 8 or 16 bytes");
    set_e<1, E0>(r, u32(*p));
  }
}
template <int W, int VL, int K, int NW, int HINT = 0>
__device__ __forceinline__ void store_vec(const u32 (&r)[NW], u8* p) {
  constexpr int VB = W << VL;
  constexpr int E0 = K << VL;
  if constexpr (VB == 16) {
    stg_v4<HINT>(p, r[E0 * W / 4 + 0], r[E0 * W / 4 + 1], r[E0 * W / 4 + 2], r[E0 * W / 4 + 3]);
  } else if constexpr (VB == 8) {
    stg_v2<HINT>(p, r[E0 * W / 4 + 0], r[E0 * W / 4 + 1]);
  } else if constexpr (VB == 4) {
    stg_b32<HINT>(p, r[E0 * W / 4]);
  } else if constexpr (VB == 2) {
    *reinterpret_cast<u16*>(p) = u16(get_e<2, E0 * W / 2>(r));
  } else {
    static_assert(VB == 1, "global vector width must be 1, 2, 4, 8 or 16 bytes");
    *p = u8(get_e<1, E0>(r));
  }
}

// Byte offset (within the tile) of thread-local vector K: XOR of the per-register-bit
// columns (compile time).
template <class P, int K> struct LdOff {
  static constexpr u64 value() {
    u64 o = 0;
    for (int b = P::VLD; b < P::R; ++b) if (((K << P::VLD) >> b) & 1) o ^= P::LD_COL[b];
    return o;
  }
};
template <class P, int K> struct StOff {
  static constexpr u64 value() {
    u64 o = 0;
    for (int b = P::VST; b < P::R; ++b) if (((K << P::VST) >> b) & 1) o ^= P::ST_COL[b];
    return o;
  }
};

// In-vector XOR of thread-local vector K (XOR-copy plans, LD_INVEC): the element XOR
// its register bits contribute inside the aligned src vector (compile time).
template <class P, int K> struct LdLo {
  static constexpr u32 value() {
    u32 c = 0;
    for (int b = P::VLD; b < P::R; ++b) if (((K << P::VLD) >> b) & 1) c ^= P::LD_LO[b];
    return c;
  }
};

// Permute the 2^VL elements of W bytes of vector K by element index XOR c (runtime):
// out element e = in element e ^ c.  Word-index bits by conditional swaps (selp),
// sub-word bits by one byte permute (prmt) per word.  Vectors of >= 4 bytes.
template <int W, int VL, int K, int NW>
__device__ __forceinline__ void xor_perm_vec(u32 (&r)[NW], u32 c) {
  constexpr int VB = W << VL;
  static_assert(VB >= 4, "in-vector XOR needs vectors of >= 4 bytes");
  constexpr int NWV = VB / 4;                  // words in the vector
  constexpr int EPW = W < 4 ? 4 / W : 1;       // elements per word
  constexpr int SH = EPW == 4 ? 2 : (EPW == 2 ? 1 : 0);
  constexpr int W0 = (K << VL) * W / 4;        // first word of the vector
  if constexpr (SH > 0) {
    const u32 ce = c & (EPW - 1);
    u32 sel;
    if constexpr (W == 2) sel = ce ? 0x1032u : 0x3210u;
    else sel = (0u ^ ce) | ((1u ^ ce) << 4) | ((2u ^ ce) << 8) | ((3u ^ ce) << 12);
    static_for<NWV>([&](auto q) {
      constexpr int Q = decltype(q)::value;
      r[W0 + Q] = __byte_perm(r[W0 + Q], 0u, sel);
    });
  }
  const u32 cw = c >> SH;
  static_for<(NWV > 1 ? (NWV == 2 ? 1 : 2) : 0)>([&](auto t) {
    constexpr int T = decltype(t)::value;
    const bool p = (cw >> T) & 1u;
    static_for<NWV>([&](auto j) {
      constexpr int J = decltype(j)::value;
      constexpr int JX = J ^ (1 << T);
      if constexpr (JX > J) {
        const u32 a = r[W0 + J], b = r[W0 + JX];
        r[W0 + J] = p ? b : a;
        r[W0 + JX] = p ? a : b;
      }
    });
  });
}

// Per-thread base from the lane / warp columns (runtime lane, warp).
template <class P, bool LD>
__device__ __forceinline__ u64 thread_base(u32 lane, u32 warp) {
  u64 o = 0;
  static_for<5>([&](auto t) {
    constexpr int T = decltype(t)::value;
    u64 c;
    if constexpr (LD) c = P::LD_COL[P::R + T]; else c = P::ST_COL[P::R + T];
    if ((lane >> T) & 1) o ^= c;
  });
  static_for<P::WB>([&](auto t) {
    constexpr int T = decltype(t)::value;
    u64 c;
    if constexpr (LD) c = P::LD_COL[P::R + 5 + T]; else c = P::ST_COL[P::R + 5 + T];
    if ((warp >> T) & 1) o ^= c;
  });
  return o;
}

template <class P, bool LD>
__device__ __forceinline__ u64 tile_base(u64 t) {
  if constexpr (P::GRID_CONTIG) {
    if constexpr (LD) return t << P::GRID_LD_SHIFT; else return t << P::GRID_ST_SHIFT;
  } else {
    u64 o = 0;
    static_for<P::G>([&](auto g) {
      constexpr int Gi = decltype(g)::value;
      u64 c;
      if constexpr (LD) c = P::GRID_LD[Gi]; else c = P::GRID_ST[Gi];
      if ((t >> Gi) & 1) o ^= c;
    });
    return o;
  }
}

// ------------------------------------------------------------------ exchanges
// a6 REGPERM: out slot e <- in slot PERM[e]; free renaming for W = 4.
template <class P>
__device__ __forceinline__ void xchg_regperm(const u32 (&r)[P::NW], u32 (&o)[P::NW]) {
  static_for<(1 << P::R)>([&](auto e) {
    constexpr int E = decltype(e)::value;
    set_e<P::W, E>(o, get_e<P::W, P::PERM[E]>(r));
  });
}

// Conditional-swap network: slot j <-> slot j^X[s] when parity(lane & MASK[s]).
template <class P, bool PRE>
__device__ __forceinline__ void xor_net(u32 (&r)[P::NW], u32 lane) {
  constexpr int NST = PRE ? P::NPRE : P::NPOST;
  static_for<NST>([&](auto s) {
    constexpr int S = decltype(s)::value;
    constexpr u32 MASK = PRE ? P::PRE_LMASK[S] : P::POST_LMASK[S];
    constexpr int X = PRE ? P::PRE_X[S] : P::POST_X[S];
    const bool p = __popc(lane & MASK) & 1;
    static_for<P::NSLOT>([&](auto j) {
      constexpr int J = decltype(j)::value;
      constexpr int K = J ^ X;
      if constexpr (K > J) {
        static_for<P::UW>([&](auto q) {
          constexpr int Q = decltype(q)::value;
          const u32 a = r[J * P::UW + Q], b = r[K * P::UW + Q];
          r[J * P::UW + Q] = p ? b : a;
          r[K * P::UW + Q] = p ? a : b;
        });
      }
    });
  });
}

// a7 SHUFFLE: pre-permutation (slot ^= M·lane), 2^|R| rounds of
// shfl.sync.idx moving one 32-bit unit each, static renaming, post-permutation.
template <class P>
__device__ __forceinline__ void xchg_shuffle(u32 (&r)[P::NW], u32 (&o)[P::NW], u32 lane) {
  xor_net<P, true>(r, lane);
  u32 lx = 0;
  static_for<5>([&](auto t) {
    constexpr int T = decltype(t)::value;
    if ((lane >> T) & 1) lx ^= P::SRC_LANE_COL[T];
  });
  static_for<P::ROUNDS>([&](auto rr) {
    constexpr int RR = decltype(rr)::value;
    constexpr int S = P::SEND_SLOT[RR];
    const int sl = int(P::SRC_LANE0[RR] ^ lx);
    static_for<P::UW>([&](auto q) {
      constexpr int Q = decltype(q)::value;
      r[S * P::UW + Q] = __shfl_sync(0xffffffffu, r[S * P::UW + Q], sl);
    });
  });
  static_for<P::ROUNDS>([&](auto rr) {
    constexpr int RR = decltype(rr)::value;
    static_for<P::UW>([&](auto q) {
      constexpr int Q = decltype(q)::value;
      o[P::RECV_SLOT[RR] * P::UW + Q] = r[P::SEND_SLOT[RR] * P::UW + Q];
    });
  });
  xor_net<P, false>(o, lane);
}

// Shared-memory vector access of 2^SV elements (SV = |Vec|) at element offset off.
template <int W, int SV>
__device__ __forceinline__ void sts_vec(u32 addr, const u32* v) {
  constexpr int VB = W << SV;
  if constexpr (VB == 16)
    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(addr), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]) : "memory");
  else if constexpr (VB == 8)
    asm volatile("st.shared.v2.u32 [%0], {%1,%2};" ::"r"(addr), "r"(v[0]), "r"(v[1]) : "memory");
  else if constexpr (VB == 4)
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(v[0]) : "memory");
  else if constexpr (VB == 2)
    asm volatile("st.shared.u16 [%0], %1;" ::"r"(addr), "h"(u16(v[0])) : "memory");
  else {
    static_assert(VB == 1, "shared vector width must be 1, 2, 4, 8 or 16 bytes");
    asm volatile("st.shared.u8 [%0], %1;" ::"r"(addr), "r"(v[0]) : "memory");
  }
}
template <int W, int SV>
__device__ __forceinline__ void lds_vec(u32 addr, u32* v) {
  constexpr int VB = W << SV;
  if constexpr (VB == 16)
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(addr) : "memory");
  else if constexpr (VB == 8)
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(addr) : "memory");
  else if constexpr (VB == 4)
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v[0]) : "r"(addr) : "memory");
  else if constexpr (VB == 2) {
    u16 h;
    asm volatile("ld.shared.u16 %0, [%1];" : "=h"(h) : "r"(addr) : "memory");
    v[0] = h;
  } else {
    static_assert(VB == 1, "shared vector width must be 1, 2, 4, 8 or 16 bytes");
    u32 b;
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(b) : "r"(addr) : "memory");
    v[0] = b & 0xffu;
  }
}

template <class P, int K, bool ST> struct SmVec {
  // register slot of vector K's element 0 (non-Vec register bits enumerate K) and
  // its smem element offset (M^{-1} ∘ L of those bits)
  static constexpr int base_slot() {
    int s = 0, k = K, t = 0;
    for (int b = 0; b < P::R; ++b) {
      bool isvec = false;
      for (int i = 0; i < P::SV; ++i) if ((ST ? P::VSLOT_LD[i] : P::VSLOT_ST[i]) == b) isvec = true;
      if (isvec) continue;
      if ((k >> t) & 1) s |= 1 << b;
      ++t;
    }
    return s;
  }
  static constexpr u64 off() {
    u64 o = 0;
    int s = base_slot();
    for (int b = 0; b < P::R; ++b) if ((s >> b) & 1) o ^= (ST ? P::SMOFF_LD[b] : P::SMOFF_ST[b]);
    return o;
  }
  template <int I> static constexpr int slot() {
    int s = base_slot();
    for (int i = 0; i < P::SV; ++i) if ((I >> i) & 1) s ^= 1 << (ST ? P::VSLOT_LD[i] : P::VSLOT_ST[i]);
    return s;
  }
};

template <class P, bool ST>
__device__ __forceinline__ u32 smem_thread_base(u32 lane, u32 warp) {
  u32 o = 0;
  static_for<5>([&](auto t) {
    constexpr int T = decltype(t)::value;
    constexpr u32 c = u32(ST ? P::SMOFF_LD[P::R + T] : P::SMOFF_ST[P::R + T]);
    if ((lane >> T) & 1) o ^= c;
  });
  static_for<P::WB>([&](auto t) {
    constexpr int T = decltype(t)::value;
    constexpr u32 c = u32(ST ? P::SMOFF_LD[P::R + 5 + T] : P::SMOFF_ST[P::R + 5 + T]);
    if ((warp >> T) & 1) o ^= c;
  });
  return o;
}

// a8 SMEM: st.shared through M^{-1}∘L_ld, barrier,
// ld.shared through M^{-1}∘L_st; M is the optimal swizzle (conflict-free).
template <class P>
__device__ __forceinline__ void smem_write(const u32 (&r)[P::NW], u32 lane, u32 warp, u32 sbase) {
  constexpr int VE = 1 << P::SV;
  constexpr int VW = (P::W * VE + 3) / 4;
  u32 tst = smem_thread_base<P, true>(lane, warp);
  // NOHOIST (linear tiles): an opaque copy per call keeps the 2^R XOR-combined smem
  // addresses out of the tile loop — hoisted as loop invariants they outgrow the register
  // file and spill (measured: 255 registers + local-memory stack)
  if constexpr (P::NOHOIST) asm volatile("" : "+r"(tst));
  static_for<(1 << (P::R - P::SV))>([&](auto k) {
    constexpr int K = decltype(k)::value;
    u32 v[VW > 0 ? VW : 1];
    static_for<VW>([&](auto q) { v[decltype(q)::value] = 0; });
    static_for<VE>([&](auto i) {
      constexpr int I = decltype(i)::value;
      constexpr int S = SmVec<P, K, true>::template slot<I>();
      set_e<P::W, I>(v, get_e<P::W, S>(r));
    });
    constexpr u32 off = u32(SmVec<P, K, true>::off());
    sts_vec<P::W, P::SV>(sbase + (tst ^ off) * P::W, v);
  });
}
template <class P>
__device__ __forceinline__ void smem_read(u32 (&o)[P::NW], u32 lane, u32 warp, u32 sbase) {
  constexpr int VE = 1 << P::SV;
  constexpr int VW = (P::W * VE + 3) / 4;
  u32 tld = smem_thread_base<P, false>(lane, warp);
  if constexpr (P::NOHOIST) asm volatile("" : "+r"(tld));
  static_for<(1 << (P::R - P::SV))>([&](auto k) {
    constexpr int K = decltype(k)::value;
    u32 v[VW > 0 ? VW : 1];
    constexpr u32 off = u32(SmVec<P, K, false>::off());
    lds_vec<P::W, P::SV>(sbase + (tld ^ off) * P::W, v);
    static_for<VE>([&](auto i) {
      constexpr int I = decltype(i)::value;
      constexpr int S = SmVec<P, K, false>::template slot<I>();
      set_e<P::W, S>(o, get_e<P::W, I>(v));
    });
  });
}
// stmatrix / ldmatrix sides (Thm 5.1): M^{-1}∘L is divisible by the tile
// id_k^{Reg,Off} × id_2^{Thr,Off} (k = log2(4/W)): a 32-bit word of k register bits
// and lanes 0, 1 make one 16-byte row of an 8x8 b16 matrix, lanes 2-4 its 8 rows
// (SMI 1); or, transposed (SMI 2, W = 2), lanes 2-4 make the row and (word bit,
// lane 0, lane 1) its rows.  Up to two further register bits select the matrix
// (.x1/.x2/.x4); lane 8m + r supplies the address of row r of matrix m.
// ST = true: the store side (L_ld data, stmatrix); false: the load side (ldmatrix).
template <class P, bool ST> struct Mx {
  static constexpr int KIND = ST ? P::SMI_LD : P::SMI_ST;
  static constexpr int NWB = P::NMW;
  static constexpr int NSEL = ST ? P::NMSEL_LD : P::NMSEL_ST;
  static constexpr int NOTHER = P::R - NWB - NSEL;
  static constexpr int wordbit(int i) { return ST ? P::MWORD_LD[i] : P::MWORD_ST[i]; }
  static constexpr int selbit(int j) { return ST ? P::MSEL_LD[j] : P::MSEL_ST[j]; }
  static constexpr u64 smoff(int b) { return ST ? P::SMOFF_LD[b] : P::SMOFF_ST[b]; }
  static constexpr bool special(int b) {
    for (int i = 0; i < NWB; ++i) if (wordbit(i) == b) return true;
    for (int j = 0; j < NSEL; ++j) if (selbit(j) == b) return true;
    return false;
  }
  // register slot of element i of matrix m in instruction k
  static constexpr int slot(int k, int m, int i) {
    int s = 0, t = 0;
    for (int b = 0; b < P::R; ++b) {
      if (special(b)) continue;
      if ((k >> t) & 1) s |= 1 << b;
      ++t;
    }
    for (int j = 0; j < NSEL; ++j) if ((m >> j) & 1) s |= 1 << selbit(j);
    for (int q = 0; q < NWB; ++q) if ((i >> q) & 1) s |= 1 << wordbit(q);
    return s;
  }
  // smem element offset of instruction k (its non-special register bits)
  static constexpr u64 off(int k) {
    u64 o = 0;
    int t = 0;
    for (int b = 0; b < P::R; ++b) {
      if (special(b)) continue;
      if ((k >> t) & 1) o ^= smoff(b);
      ++t;
    }
    return o;
  }
  // the three bits addressing the rows of a matrix
  static constexpr u64 rowoff(int t) {
    return KIND == 1 ? smoff(P::R + 2 + t) : (t == 0 ? smoff(wordbit(0)) : smoff(P::R + t - 1));
  }
};

// Row address supplied by this lane: row (lane & 7) of matrix (lane >> 3).
template <class P, bool ST>
__device__ __forceinline__ u32 mat_thread_base(u32 lane, u32 warp) {
  typedef Mx<P, ST> X;
  u32 o = 0;
  static_for<3>([&](auto t) {
    constexpr int T = decltype(t)::value;
    if ((lane >> T) & 1) o ^= u32(X::rowoff(T));
  });
  static_for<X::NSEL>([&](auto j) {
    constexpr int J = decltype(j)::value;
    if ((lane >> (3 + J)) & 1) o ^= u32(X::smoff(X::selbit(J)));
  });
  static_for<P::WB>([&](auto t) {
    constexpr int T = decltype(t)::value;
    if ((warp >> T) & 1) o ^= u32(X::smoff(P::R + 5 + T));
  });
  return o;
}

template <int NSEL, bool TRANS>
__device__ __forceinline__ void stsm(u32 addr, const u32* v) {
  if constexpr (NSEL == 2) {
    if constexpr (TRANS)
      asm volatile("stmatrix.sync.aligned.m8n8.x4.trans.shared.b16 [%0], {%1,%2,%3,%4};"
                   ::"r"(addr), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]) : "memory");
    else
      asm volatile("stmatrix.sync.aligned.m8n8.x4.shared.b16 [%0], {%1,%2,%3,%4};"
                   ::"r"(addr), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]) : "memory");
  } else if constexpr (NSEL == 1) {
    if constexpr (TRANS)
      asm volatile("stmatrix.sync.aligned.m8n8.x2.trans.shared.b16 [%0], {%1,%2};" ::"r"(addr), "r"(v[0]), "r"(v[1]) : "memory");
    else
      asm volatile("stmatrix.sync.aligned.m8n8.x2.shared.b16 [%0], {%1,%2};" ::"r"(addr), "r"(v[0]), "r"(v[1]) : "memory");
  } else {
    if constexpr (TRANS)
      asm volatile("stmatrix.sync.aligned.m8n8.x1.trans.shared.b16 [%0], {%1};" ::"r"(addr), "r"(v[0]) : "memory");
    else
      asm volatile("stmatrix.sync.aligned.m8n8.x1.shared.b16 [%0], {%1};" ::"r"(addr), "r"(v[0]) : "memory");
  }
}
template <int NSEL, bool TRANS>
__device__ __forceinline__ void ldsm(u32 addr, u32* v) {
  if constexpr (NSEL == 2) {
    if constexpr (TRANS)
      asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(addr) : "memory");
    else
      asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(addr) : "memory");
  } else if constexpr (NSEL == 1) {
    if constexpr (TRANS)
      asm volatile("ldmatrix.sync.aligned.m8n8.x2.trans.shared.b16 {%0,%1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(addr) : "memory");
    else
      asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0,%1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(addr) : "memory");
  } else {
    if constexpr (TRANS)
      asm volatile("ldmatrix.sync.aligned.m8n8.x1.trans.shared.b16 {%0}, [%1];" : "=r"(v[0]) : "r"(addr) : "memory");
    else
      asm volatile("ldmatrix.sync.aligned.m8n8.x1.shared.b16 {%0}, [%1];" : "=r"(v[0]) : "r"(addr) : "memory");
  }
}

template <class P>
__device__ __forceinline__ void smem_write_mat(const u32 (&r)[P::NW], u32 lane, u32 warp, u32 sbase) {
  typedef Mx<P, true> X;
  const u32 tb = mat_thread_base<P, true>(lane, warp);
  static_for<(1 << X::NOTHER)>([&](auto k) {
    constexpr int K = decltype(k)::value;
    u32 v[1 << X::NSEL];
    static_for<(1 << X::NSEL)>([&](auto m) {
      constexpr int M = decltype(m)::value;
      if constexpr (P::W == 4) {
        v[M] = r[X::slot(K, M, 0)];
      } else {
        u32 word = 0;
        static_for<(1 << X::NWB)>([&](auto i) {
          constexpr int I = decltype(i)::value;
          word |= get_e<P::W, X::slot(K, M, I)>(r) << (8 * P::W * I);
        });
        v[M] = word;
      }
    });
    stsm<X::NSEL, X::KIND == 2>(sbase + (tb ^ u32(X::off(K))) * P::W, v);
  });
}
template <class P>
__device__ __forceinline__ void smem_read_mat(u32 (&o)[P::NW], u32 lane, u32 warp, u32 sbase) {
  typedef Mx<P, false> X;
  const u32 tb = mat_thread_base<P, false>(lane, warp);
  static_for<(1 << X::NOTHER)>([&](auto k) {
    constexpr int K = decltype(k)::value;
    u32 v[1 << X::NSEL];
    ldsm<X::NSEL, X::KIND == 2>(sbase + (tb ^ u32(X::off(K))) * P::W, v);
    static_for<(1 << X::NSEL)>([&](auto m) {
      constexpr int M = decltype(m)::value;
      if constexpr (P::W == 4) {
        o[X::slot(K, M, 0)] = v[M];
      } else {
        static_for<(1 << X::NWB)>([&](auto i) {
          constexpr int I = decltype(i)::value;
          set_e<P::W, X::slot(K, M, I)>(o, (v[M] >> (8 * P::W * I)) & (P::W == 2 ? 0xffffu : 0xffu));
        });
      }
    });
  });
}

template <class P>
__device__ __forceinline__ void smem_store(const u32 (&r)[P::NW], u32 lane, u32 warp, u32 sbase) {
  if constexpr (P::SMI_LD != 0) smem_write_mat<P>(r, lane, warp, sbase);
  else smem_write<P>(r, lane, warp, sbase);
}
template <class P>
__device__ __forceinline__ void smem_load(u32 (&o)[P::NW], u32 lane, u32 warp, u32 sbase) {
  if constexpr (P::SMI_ST != 0) smem_read_mat<P>(o, lane, warp, sbase);
  else smem_read<P>(o, lane, warp, sbase);
}
template <class P>
__device__ __forceinline__ void xchg_smem(const u32 (&r)[P::NW], u32 (&o)[P::NW], u32 lane, u32 warp, u32 sbase) {
  smem_store<P>(r, lane, warp, sbase);
  __syncthreads();
  smem_load<P>(o, lane, warp, sbase);
}

// ------------------------------------------------------------------ TMA bulk copies
// cp.async.bulk (SASS UBLKCP) global -> shared, completion tracked by an mbarrier
// (expect_tx / complete_tx), the Blackwell async-copy pipeline.
__device__ __forceinline__ void mbar_init(u32 bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(u32 bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(u32 dst, const void* src, u32 bytes, u32 bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(u32 bar, u32 parity) {
  u32 ok = 0;
  do {
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                 "selp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
  } while (!ok);
}

// shared -> global bulk copy (SASS UBLKCP), completion by bulk async-group
__device__ __forceinline__ void bulk_s2g(void* dst, u32 src, u32 bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}


// One w-byte element to / from shared memory (broadcast dst-order stores).
template <int W> __device__ __forceinline__ void sts_elem(u32 addr, u32 v) {
  if constexpr (W == 4) asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
  else if constexpr (W == 2) asm volatile("st.shared.u16 [%0], %1;" ::"r"(addr), "h"(u16(v)) : "memory");
  else { static_assert(W == 1, "element width"); asm volatile("st.shared.u8 [%0], %1;" ::"r"(addr), "r"(v) : "memory"); }
}
template <int W> __device__ __forceinline__ u32 lds_elem(u32 addr) {
  u32 v;
  if constexpr (W == 4) asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  else if constexpr (W == 2) { u16 h; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(h) : "r"(addr) : "memory"); v = h; }
  else { static_assert(W == 1, "element width"); asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(addr) : "memory"); v &= 0xffu; }
  return v;
}
// compile-time XOR of a column table over the set bits of an index
template <class P, int E> struct BcW {   // smem element offset of load register slot E
  static constexpr u32 value() { u32 o = 0; for (int b = 0; b < P::R; ++b) if ((E >> b) & 1) o ^= u32(P::BC_SMW[b]); return o; }
};
template <class P, int E> struct BcR {   // smem element offset of store-vector element E
  static constexpr u32 value() { u32 o = 0; for (int b = 0; b < P::BC_V; ++b) if ((E >> b) & 1) o ^= u32(P::BC_SMR[b]); return o; }
  // the element E' < E that reads the same smem element (a replica bit of the vector)
  static constexpr int same() {
    for (int b = 0; b < P::BC_V; ++b) if (((E >> b) & 1) && P::BC_SMR[b] == 0) return E & ~(1 << b);
    return -1;
  }
};

// ------------------------------------------------------------------ tile kernel
// Programmatic dependent launch (sm_90+): the host launches every kernel with the
// programmatic-stream-serialization attribute, so a kernel's CTAs may be scheduled
// while the previous kernel in the stream drains.  Each CTA waits for the previous
// grid's memory to be visible before touching global memory, then lets the next
// grid launch (its CTAs in turn wait here), hiding launch latency and ramp.
__device__ __forceinline__ void ll_pdl_begin() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// Destination addressing of the tile kernel.  DstLocal: one buffer.  DstPeers (row
// a9 DEVICE plans executed as peer stores, §8(f) N4): the dst offset is an offset in
// the GLOBAL packed index space (local bits, then the dev bits on top); its top bits
// select the receiving rank's window (NVLink peer memory mapped into this process).
struct DstLocal {
  u8* base;
  __device__ __forceinline__ explicit DstLocal(u8* b) : base(b) {}
  __device__ __forceinline__ u8* at(u64 off) const { return base + off; }
};
#ifndef LL_MAX_PEERS
#define LL_MAX_PEERS 64
#endif
struct LLPeers {
  u8* dst[LL_MAX_PEERS];
};
template <int SHIFT>
struct DstPeers {
  const LLPeers* p;
  __device__ __forceinline__ explicit DstPeers(const LLPeers* q) : p(q) {}
  __device__ __forceinline__ u8* at(u64 off) const {
    return p->dst[off >> SHIFT] + (off & ((u64(1) << SHIFT) - 1));
  }
};

template <class D> struct IsDstLocal { static constexpr bool value = false; };
template <> struct IsDstLocal<DstLocal> { static constexpr bool value = true; };

// PEER_REG: some register / replica bit of the dst tile crosses ranks, so every
// store picks its window; otherwise one window per thread and tile.
template <class P, class Dst, bool PEER_REG = false>
__device__ __forceinline__ void ll_tile_body(const u8* __restrict__ src, Dst D, u64 ntiles, u64 tile0 = 0) {
  extern __shared__ __align__(16) u8 ll_smem[];
  ll_pdl_begin();
  const u32 lane = threadIdx.x & 31u;
  const u32 warp = threadIdx.x >> 5;
  const u64 ld_thr = thread_base<P, true>(lane, warp);
  const u64 st_thr = thread_base<P, false>(lane, warp);
  const u32 sbase = u32(__cvta_generic_to_shared(ll_smem));
  if constexpr (P::XCHG == 3 && P::ISOLATE_SMEM) {
    // Diagnostic variant (codegen env LL_ISOLATE_SMEM=1): the smem exchange alone,
    // 16 times, with no global traffic — separates true bank conflicts from L1 data
    // pipe contention with concurrent global loads in ncu's counters.
    u32 r[P::NW], o[P::NW];
    static_for<P::NW>([&](auto q) { r[decltype(q)::value] = threadIdx.x * 131u + decltype(q)::value; });
    for (int it = 0; it < 16; ++it) {
      xchg_smem<P>(r, o, lane, warp, sbase);
      __syncthreads();
      static_for<P::NW>([&](auto q) { r[decltype(q)::value] = o[decltype(q)::value] + 1u; });
    }
    if (r[0] == 0x9e3779b9u) *D.at(threadIdx.x) = u8(r[P::NW - 1]);
    return;
  }
  // a5: HBM load of a src tile (16-byte vectors; coalesced under σ_ld)
  // in-vector XOR of this thread (lane / warp columns), XOR-copy plans only
  u32 lo_thr = 0;
  if constexpr (P::LD_INVEC) {
    static_for<5>([&](auto q) {
      constexpr int T = decltype(q)::value;
      if ((lane >> T) & 1) lo_thr ^= P::LD_LO[P::R + T];
    });
    static_for<P::WB>([&](auto q) {
      constexpr int T = decltype(q)::value;
      if ((warp >> T) & 1) lo_thr ^= P::LD_LO[P::R + 5 + T];
    });
  }
  // broadcast plans: the lowest NREP_HI_BITS CTA-index bits select a group of replica
  // offsets (the replica bits above the unrolled ones are grid bits), the
  // bits above them the data tile — CTAs that load the same src tile run together, so
  // its re-reads hit L2
  constexpr u64 RGMASK = (u64(1) << P::NREP_HI_BITS) - 1;
  auto load_tile = [&](u32 (&r)[P::NW], u64 t) {
    if constexpr (P::NREP_HI_BITS > 0) t >>= P::NREP_HI_BITS;
    u64 thr = ld_thr;
    if constexpr (P::NOHOIST) asm volatile("" : "+l"(thr));   // keep per-vector addresses in the loop
    const u64 sofs = tile_base<P, true>(t) ^ thr;
    const u8* s = src + sofs;
    u32 lo = lo_thr;
    if constexpr (P::LD_INVEC) {
      static_for<P::G>([&](auto g) {
        constexpr int Gi = decltype(g)::value;
        if ((t >> Gi) & 1) lo ^= P::GRID_LD_LO[Gi];
      });
    }
    static_for<(1 << (P::R - P::VLD))>([&](auto k) {
      constexpr int K = decltype(k)::value;
      // XOR-copy plans (non-permutation Q): register and thread offsets share bits,
      // so they combine by XOR; permutation plans' bits are disjoint (immediate add)
      if constexpr (P::LD_XOR) {
        load_vec<P::W, P::VLD, K, P::NW, P::LD_L1>(r, src + (sofs ^ LdOff<P, K>::value()));
        if constexpr (P::LD_INVEC) xor_perm_vec<P::W, P::VLD, K, P::NW>(r, lo ^ LdLo<P, K>::value());
      } else {
        load_vec<P::W, P::VLD, K, P::NW, P::LD_L1>(r, s + LdOff<P, K>::value());
      }
    });
  };
  // a10: HBM store of a dst tile (and of its broadcast replicas)
  auto store_tile = [&](const u32 (&o)[P::NW], u64 t) {
    u64 thr = st_thr;
    if constexpr (P::NOHOIST) asm volatile("" : "+l"(thr));
    const u64 td = P::NREP_HI_BITS > 0 ? (t >> P::NREP_HI_BITS) : t;
    const u64 doff = tile_base<P, false>(td | tile0) ^ thr;
    auto store_reps = [&](u64 ho) {
      u8* d = D.at(doff ^ ho);
      static_for<P::NREP>([&](auto rp) {
        constexpr u64 RO = P::REP_OFF[decltype(rp)::value];
        static_for<(1 << (P::R - P::VST))>([&](auto k) {
          constexpr int K = decltype(k)::value;
          if constexpr (PEER_REG)
            store_vec<P::W, P::VST, K, P::NW, P::ST_HINT>(o, D.at((doff ^ ho) + (StOff<P, K>::value() ^ RO)));
          else
            store_vec<P::W, P::VST, K, P::NW, P::ST_HINT>(o, d + (StOff<P, K>::value() ^ RO));
        });
      });
    };
    if constexpr (P::NREP_HI_BITS == 0) {
      store_reps(0);
    } else {
      // replica bits above the unrolled ones: this CTA's group (CTA-index bits above G)
      const u32 rg = u32(t & RGMASK);
      u64 ho = 0;
      static_for<P::NREP_HI_BITS>([&](auto j) {
        constexpr int J = decltype(j)::value;
        if ((rg >> J) & 1u) ho ^= P::REP_HI[J];
      });
      store_reps(ho);
    }
  };
  if constexpr (P::XCHG == 3 && P::STAGED) {
    // Staged smem exchange (ll_plan_opts.pipe = 3): the src vectors of the next two
    // tiles stream into two raw stages by cp.async (16 bytes each, thread-slot order
    // [vector][thread]: 512 contiguous bytes per warp instruction, conflict-free), so a
    // CTA keeps two tiles of loads in flight without holding them in registers.  Each
    // thread reads back only its own slots (cp.async.wait_group is per thread), then
    // the tile takes the usual swizzled round trip.  Persistent grid (one CTA per SM).
    constexpr int NV = 1 << (P::R - P::VLD);
    constexpr u32 TB = u32(P::THREADS) * NV * 16u;
    const u32 stage0 = sbase + P::XBYTES;
    auto issue = [&](u64 t, u32 st) {
      if (t < ntiles) {
        const u64 sofs = tile_base<P, true>(t) ^ ld_thr;
        static_for<NV>([&](auto k) {
          constexpr int K = decltype(k)::value;
          const u8* g;
          if constexpr (P::LD_XOR) g = src + (sofs ^ LdOff<P, K>::value());
          else g = src + sofs + LdOff<P, K>::value();
          cp_async16(stage0 + st * TB + (u32(K) * P::THREADS + threadIdx.x) * 16u, g);
        });
      }
      cp_async_commit();   // empty groups past the end keep the group count uniform
    };
    u64 t = blockIdx.x;
    issue(t, 0);
    issue(t + gridDim.x, 1);
    for (u32 i = 0; t < ntiles; t += gridDim.x, ++i) {
      const u32 st = i & 1u;
      cp_async_wait1();    // every group but the newest: tile t's vectors have landed
      u32 r[P::NW];
      static_for<NV>([&](auto k) {
        constexpr int K = decltype(k)::value;
        lds_v4(stage0 + st * TB + (u32(K) * P::THREADS + threadIdx.x) * 16u, r[4 * K], r[4 * K + 1], r[4 * K + 2],
               r[4 * K + 3]);
      });
      if constexpr (P::LD_INVEC) {
        u32 lo = lo_thr;
        static_for<P::G>([&](auto g) {
          constexpr int Gi = decltype(g)::value;
          if ((t >> Gi) & 1) lo ^= P::GRID_LD_LO[Gi];
        });
        static_for<NV>([&](auto k) {
          constexpr int K = decltype(k)::value;
          xor_perm_vec<P::W, P::VLD, K, P::NW>(r, lo ^ LdLo<P, K>::value());
        });
      }
      smem_store<P>(r, lane, warp, sbase);   // r consumed: this thread's stage reads are done
      issue(t + 2 * u64(gridDim.x), st);
      __syncthreads();
      u32 o[P::NW];
      static_for<P::NW>([&](auto q) { o[decltype(q)::value] = 0; });
      smem_load<P>(o, lane, warp, sbase);
      store_tile(o, t);
      __syncthreads();   // exchange buffer reuse by the next tile
    }
    cp_async_wait0();
    return;
  }
  if constexpr (P::BCAST) {
    // Broadcast stores in dst order (TilePlan::bcast): the data tile goes to
    // smem in dst-data order; every thread then reads whole 16-byte dst vectors along
    // the store tile U (replica bits add 0 to the smem offset: broadcast reads of the same
    // element) and stores them with 512 contiguous bytes per warp instruction; replica
    // bits above U are unrolled offsets / grid groups as in store_tile.
    u32 thr_w = 0, thr_r = 0;
    u64 thr_s = 0;
    static_for<5>([&](auto q) {
      constexpr int T = decltype(q)::value;
      if ((lane >> T) & 1) { thr_w ^= u32(P::BC_SMW[P::R + T]); thr_r ^= u32(P::BC_SMR[P::BC_V + T]); thr_s ^= P::BC_ST[P::BC_V + T]; }
    });
    static_for<P::WB>([&](auto q) {
      constexpr int T = decltype(q)::value;
      if ((warp >> T) & 1) { thr_w ^= u32(P::BC_SMW[P::R + 5 + T]); thr_r ^= u32(P::BC_SMR[P::BC_V + 5 + T]); thr_s ^= P::BC_ST[P::BC_V + 5 + T]; }
    });
    constexpr int KB0 = P::BC_V + 5 + P::WB;   // first U bit of the per-thread vector index
    for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x) {
      u32 r[P::NW];
      load_tile(r, t);
      static_for<(1 << P::R)>([&](auto e) {
        constexpr int E = decltype(e)::value;
        sts_elem<P::W>(sbase + (thr_w ^ BcW<P, E>::value()) * u32(P::W), get_e<P::W, E>(r));
      });
      __syncthreads();
      const u64 td = P::NREP_HI_BITS > 0 ? (t >> P::NREP_HI_BITS) : t;
      u64 ho = 0;
      if constexpr (P::NREP_HI_BITS > 0) {
        const u32 rg = u32(t & RGMASK);
        static_for<P::NREP_HI_BITS>([&](auto j) {
          constexpr int J = decltype(j)::value;
          if ((rg >> J) & 1u) ho ^= P::REP_HI[J];
        });
      }
      const u64 dbase = (tile_base<P, false>(td | tile0) ^ thr_s) ^ ho;
#pragma unroll 4
      for (u32 k = 0; k < (1u << P::BC_NK); ++k) {
        u32 kr = 0;
        u64 ks = 0;
        static_for<P::BC_NK>([&](auto j) {
          constexpr int J = decltype(j)::value;
          if ((k >> J) & 1u) { kr ^= u32(P::BC_SMR[KB0 + J]); ks ^= P::BC_ST[KB0 + J]; }
        });
        u32 v[4] = {0u, 0u, 0u, 0u};
        u32 ev[1 << P::BC_V];
        static_for<(1 << P::BC_V)>([&](auto e) {
          constexpr int E = decltype(e)::value;
          if constexpr (BcR<P, E>::same() >= 0) ev[E] = ev[BcR<P, E>::same()];
          else ev[E] = lds_elem<P::W>(sbase + (thr_r ^ kr ^ BcR<P, E>::value()) * u32(P::W));
          set_e<P::W, E>(v, ev[E]);
        });
        // replica offsets are disjoint from the tile / thread / vector bits: one base
        // pointer plus compile-time offsets (immediates, no per-store address registers
        // held by in-flight stores)
        u8* const pv = D.at(dbase ^ ks);
        static_for<P::NREP>([&](auto rp) {
          constexpr u64 RO = P::REP_OFF[decltype(rp)::value];
          store_vec<P::W, P::BC_V, 0, 4, P::ST_HINT>(v, pv + RO);
        });
      }
      __syncthreads();   // smem reuse by the next tile
    }
    return;
  }
  if constexpr (P::XCHG == 3 && P::BULK) {
    // Bulk-staged smem exchange (ll_plan_opts.pipe = 4, LL_PIPE=bulk): the CTA tile is
    // contiguous in src-packed order, so one cp.async.bulk per tile (the TMA engine,
    // not the LSU) streams it into NS raw stages, completion on an mbarrier, NS - 1 tiles
    // ahead.  Threads read their 16-byte vectors from the stage (lanes on consecutive
    // vectors: conflict-free), then the swizzled round trip.  With BULK_ST (pipe = 5)
    // the dst tile (contiguous in dst-packed order) is written back into the exchange
    // buffer in packed order and leaves by one bulk shared -> global copy: the LSU then
    // carries shared-memory traffic only, so ncu's bank-conflict counters measure the
    // exchange alone.
    constexpr u32 TB = u32(1) << P::TILE_LOG2B;
    constexpr u32 NS = P::STAGES;
    constexpr bool BST = P::BULK_ST && IsDstLocal<Dst>::value;   // peer windows: STG stores
    const u32 stage0 = sbase + P::XBYTES;
    const u32 bar0 = stage0 + NS * TB;
    if (threadIdx.x == 0) {
      for (u32 q = 0; q < NS; ++q) mbar_init(bar0 + 8 * q, 1);
      mbar_fence_init();
    }
    __syncthreads();
    auto issue = [&](u64 tq, u32 q) {
      mbar_expect_tx(bar0 + 8 * q, TB);
      bulk_g2s(stage0 + q * TB, src + tile_base<P, true>(tq), TB, bar0 + 8 * q);
    };
    if (threadIdx.x == 0)
      for (u32 q = 0; q + 1 < NS; ++q)
        if (blockIdx.x + u64(q) * gridDim.x < ntiles) issue(blockIdx.x + u64(q) * gridDim.x, q);
    u32 i = 0;
    for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
      const u32 st = i % NS;
      const u64 tn = t + u64(NS - 1) * gridDim.x;
      if (threadIdx.x == 0 && tn < ntiles) {
        fence_proxy_async();
        issue(tn, (i + NS - 1) % NS);
      }
      mbar_wait(bar0 + 8 * st, (i / NS) & 1u);
      u32 r[P::NW];
      const u32 tb = stage0 + st * TB + u32(ld_thr);
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        load_vec_s<P::W, P::VLD, K, P::NW>(r, tb + u32(LdOff<P, K>::value()));
      });
      if constexpr (BST) {
        // the previous tile's bulk store has finished reading the exchange buffer
        if (threadIdx.x == 0) bulk_wait_read<0>();
        __syncthreads();
      }
      smem_store<P>(r, lane, warp, sbase);
      __syncthreads();   // exchange written; stage st fully read (refilled next iteration)
      u32 o[P::NW];
      static_for<P::NW>([&](auto q) { o[decltype(q)::value] = 0; });
      smem_load<P>(o, lane, warp, sbase);
      __syncthreads();   // exchange buffer free
      if constexpr (BST) {
        const u32 db = sbase + u32(st_thr);
        static_for<(1 << (P::R - P::VST))>([&](auto k) {
          constexpr int K = decltype(k)::value;
          sts_vec<P::W, P::VST>(db + u32(StOff<P, K>::value()), &o[(K << P::VST) * P::W / 4]);
        });
        fence_proxy_async();
        __syncthreads();
        if (threadIdx.x == 0) {
          bulk_s2g(D.at(tile_base<P, false>(t | tile0)), sbase, TB);
          bulk_commit();
        }
      } else {
        store_tile(o, t);
      }
    }
    if constexpr (BST) {
      if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
    return;
  }
  if constexpr (P::XCHG == 3 && P::PIPE) {
    // Software-pipelined smem exchange: once tile t sits in shared memory its
    // registers are free, so tile t + grid's loads are issued before t's smem reads
    // and HBM stores — the CTA keeps loads in flight through its store phase.
    u64 t = blockIdx.x;
    if (t >= ntiles) return;
    u32 r[P::NW];
    load_tile(r, t);
    for (; t < ntiles; t += gridDim.x) {
      smem_store<P>(r, lane, warp, sbase);
      __syncthreads();
      if (t + gridDim.x < ntiles) load_tile(r, t + gridDim.x);
      u32 o[P::NW];
      static_for<P::NW>([&](auto q) { o[decltype(q)::value] = 0; });
      smem_load<P>(o, lane, warp, sbase);
      store_tile(o, t);
      __syncthreads();   // smem reuse by the next tile
    }
    return;
  }
  for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x) {
    u32 r[P::NW];
    load_tile(r, t);
    u32 o[P::NW];
    if constexpr (P::XCHG == 0) {
      static_for<P::NW>([&](auto q) { o[decltype(q)::value] = r[decltype(q)::value]; });
    } else if constexpr (P::XCHG == 1) {
      static_for<P::NW>([&](auto q) { o[decltype(q)::value] = 0; });
      xchg_regperm<P>(r, o);
    } else if constexpr (P::XCHG == 2) {
      if constexpr (P::EPERM) {
        // thread-local element permutations: the common 32-bit unit to the lowest
        // register bits before the shuffle, the store order after it
        u32 r2[P::NW], o2[P::NW];
        static_for<P::NW>([&](auto q) { r2[decltype(q)::value] = 0; o[decltype(q)::value] = 0; });
        static_for<(1 << P::R)>([&](auto e) {
          constexpr int E = decltype(e)::value;
          set_e<P::W, E>(r2, get_e<P::W, P::PRE_EPERM[E]>(r));
        });
        xchg_shuffle<P>(r2, o2, lane);
        static_for<(1 << P::R)>([&](auto e) {
          constexpr int E = decltype(e)::value;
          set_e<P::W, E>(o, get_e<P::W, P::POST_EPERM[E]>(o2));
        });
      } else {
        xchg_shuffle<P>(r, o, lane);
      }
    } else {
      static_for<P::NW>([&](auto q) { o[decltype(q)::value] = 0; });
      xchg_smem<P>(r, o, lane, warp, sbase);
    }
    store_tile(o, t);
    if constexpr (P::XCHG == 3) __syncthreads();   // smem reuse by the next tile
  }
}

// ------------------------------------------------------------------ gather (a11)
// P:428-432 (G15 reading): per output slot, read idx, locate the source
// (register candidates, lane) and run 2^{|L_Reg^axis|} shuffle rounds, keeping the
// value whose candidate equals the source register.


// Shared-memory vector load of thread-local vector K (2^VL elements of W bytes).
template <int W, int VL, int K, int NW>
__device__ __forceinline__ void load_vec_s(u32 (&r)[NW], u32 addr) {
  constexpr int VB = W << VL;
  constexpr int E0 = K << VL;
  if constexpr (VB == 16) {
    lds_v4(addr, r[E0 * W / 4 + 0], r[E0 * W / 4 + 1], r[E0 * W / 4 + 2], r[E0 * W / 4 + 3]);
  } else if constexpr (VB == 8) {
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(r[E0 * W / 4]), "=r"(r[E0 * W / 4 + 1]) : "r"(addr) : "memory");
  } else if constexpr (VB == 4) {
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(r[E0 * W / 4]) : "r"(addr) : "memory");
  } else if constexpr (VB == 2) {
    u16 h;
    asm volatile("ld.shared.u16 %0, [%1];" : "=h"(h) : "r"(addr) : "memory");
    set_e<2, E0 * W / 2>(r, u32(h));
  } else {
    static_assert(VB == 1, "shared vector width must be 1, 2, 4, 8 or 16 bytes");
    u32 b;
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(b) : "r"(addr) : "memory");
    set_e<1, E0>(r, b & 0xffu);
  }
}

// ------------------------------------------------------------------ gather (a11)
// P:428-432 (G15 reading): per output slot, read idx, locate the source
// (register candidates, lane) and run 2^{|L_Reg^axis|} shuffle rounds, keeping the
// value whose candidate equals the source register; or, past the P:519 crossover,
// gather from the tile staged in shared memory.  With P::TMA the contiguous src and
// idx tiles are streamed through an mbarrier pipeline of cp.async.bulk copies.
template <class P>
__device__ __forceinline__ void ll_gather_body(const u8* __restrict__ src, const u8* __restrict__ idx,
                                               u8* __restrict__ dst, u64 ntiles) {
  extern __shared__ __align__(16) u8 ll_smem[];
  ll_pdl_begin();
  typedef typename std::conditional<P::W == 4, u32, typename std::conditional<P::W == 2, u16, u8>::type>::type ET;
  const u32 lane = threadIdx.x & 31u;
  const u32 warp = threadIdx.x >> 5;
  const u64 thr = thread_base<P, true>(lane, warp);           // element offsets (x W below)
  // axis coordinate contributed by this lane
  u32 a_lane = 0;
  static_for<5>([&](auto t) {
    constexpr int T = decltype(t)::value;
    if constexpr (P::AXIS_OF_LANE[T] >= 0) if ((lane >> T) & 1) a_lane ^= 1u << P::AXIS_OF_LANE[T];
  });
  // smem: [stages][src tile | idx tile] (TMA) | gather area (GATHER_SMEM) | mbarriers
  constexpr u32 NE = u32(1) << (P::R + 5 + P::WB);          // tile elements
  constexpr u32 TBS = NE * P::W, TBI = NE * 4, TBST = TBS + TBI;
  constexpr u32 NS = P::TMA ? P::STAGES : 0;
  const u32 sbase = u32(__cvta_generic_to_shared(ll_smem));
  const u32 bar0 = sbase + NS * TBST + (P::GATHER_SMEM ? TBS : 0);
  ET* sm = reinterpret_cast<ET*>(ll_smem + NS * TBST);
  u32 sthr = 0;
  if constexpr (P::GATHER_SMEM) {
    static_for<5>([&](auto t) {
      constexpr int T = decltype(t)::value;
      if ((lane >> T) & 1) sthr ^= P::SMOFF[P::R + T];
    });
    static_for<P::WB>([&](auto t) {
      constexpr int T = decltype(t)::value;
      if ((warp >> T) & 1) sthr ^= P::SMOFF[P::R + 5 + T];
    });
  }
  auto issue = [&](u64 tq, u32 q) {
    mbar_expect_tx(bar0 + 8 * q, TBST);
    const u64 eb = tile_base<P, true>(tq);
    bulk_g2s(sbase + q * TBST, src + eb * P::W, TBS, bar0 + 8 * q);
    bulk_g2s(sbase + q * TBST + TBS, idx + eb * 4, TBI, bar0 + 8 * q);
  };
  if constexpr (P::TMA) {
    if (threadIdx.x == 0) {
      for (u32 q = 0; q < NS; ++q) mbar_init(bar0 + 8 * q, 1);
      mbar_fence_init();
    }
    __syncthreads();
    if (threadIdx.x == 0)
      for (u32 q = 0; q + 1 < NS; ++q)
        if (blockIdx.x + u64(q) * gridDim.x < ntiles) issue(blockIdx.x + u64(q) * gridDim.x, q);
  }
  u32 i = 0;
  for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
    const u64 eoff = tile_base<P, true>(t) ^ thr;
    u32 r[P::NW];
    u32 ix[1 << P::R];
    if constexpr (P::TMA) {
      const u32 st = i % NS;
      const u64 tn = t + u64(NS - 1) * gridDim.x;
      if (threadIdx.x == 0 && tn < ntiles) {
        // TMA_STORE: the previous tile's bulk store read out the stage being refilled
        if constexpr (P::TMA_STORE) bulk_wait_read<0>();
        fence_proxy_async();
        issue(tn, (i + NS - 1) % NS);
      }
      mbar_wait(bar0 + 8 * st, (i / NS) & 1u);
      const u32 ts = sbase + st * TBST;
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        load_vec_s<P::W, P::VLD, K>(r, ts + u32((thr ^ LdOff<P, K>::value()) * P::W));
        load_vec_s<4, P::VLD, K>(ix, ts + TBS + u32((thr ^ LdOff<P, K>::value()) * 4));
      });
    } else {
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        load_vec<P::W, P::VLD, K, P::NW, P::LD_L1>(r, src + (eoff ^ LdOff<P, K>::value()) * P::W);
        load_vec<4, P::VLD, K, (1 << P::R), P::LD_L1>(ix, idx + (eoff ^ LdOff<P, K>::value()) * 4);
      });
    }
    u32 o[P::NW];
    static_for<P::NW>([&](auto q) { o[decltype(q)::value] = 0; });
    if constexpr (P::GATHER_SMEM) {
      // stage the tile in logical order (16-byte vectors where the thread's vector
      // registers are logically consecutive: whole 128 B lines per 8 lanes, no bank
      // conflicts), then every output reads its source element
      if constexpr (P::SMV > 0) {
        constexpr int VE = 1 << P::SMV, VW = (P::W * VE + 3) / 4;
        const u32 smb = u32(__cvta_generic_to_shared(sm));
        static_for<(1 << (P::R - P::SMV))>([&](auto k) {
          constexpr int E0 = decltype(k)::value << P::SMV;
          u32 v[VW];
          static_for<VW>([&](auto q) { v[decltype(q)::value] = 0; });
          static_for<VE>([&](auto ii) {
            constexpr int I = decltype(ii)::value;
            set_e<P::W, I>(v, get_e<P::W, E0 + I>(r));
          });
          sts_vec<P::W, P::SMV>(smb + (sthr ^ P::template smoff_of_slot<E0>()) * P::W, v);
        });
      } else {
        static_for<(1 << P::R)>([&](auto e) {
          constexpr int E = decltype(e)::value;
          sm[sthr ^ P::template smoff_of_slot<E>()] = ET(get_e<P::W, E>(r));
        });
      }
      __syncthreads();
      static_for<(1 << P::R)>([&](auto e) {
        constexpr int E = decltype(e)::value;
        const u32 kidx = ix[E] & ((1u << P::KBITS) - 1u);
        u32 off = (sthr ^ P::template smoff_of_slot<E>()) & ~P::AXMASK;
        static_for<P::KBITS>([&](auto tt) {
          constexpr int T = decltype(tt)::value;
          off |= ((kidx >> T) & 1u) << P::AXPOS[T];
        });
        set_e<P::W, E>(o, u32(sm[off]));
      });
    } else {
      static_for<(1 << P::R)>([&](auto e) {
        constexpr int E = decltype(e)::value;
        // axis coordinate of slot E's element and its candidate part
        constexpr u32 a_reg = P::template axis_of_slot<E>();
        const u32 kidx = ix[E] & ((1u << P::KBITS) - 1u);
        const u32 dlt = kidx ^ (a_reg ^ a_lane);
        u32 sl = lane, ct = 0;
        static_for<P::KBITS>([&](auto tt) {
          constexpr int T = decltype(tt)::value;
          const u32 bit = (dlt >> T) & 1u;
          if constexpr (P::AXIS_LANE_POS[T] >= 0) sl ^= bit << P::AXIS_LANE_POS[T];
          if constexpr (P::AXIS_CAND_POS[T] >= 0) ct ^= bit << P::AXIS_CAND_POS[T];
        });
        ct ^= P::template cand_of_slot<E>();
        u32 res = 0;
        static_for<(1 << P::CBITS)>([&](auto c) {
          constexpr int C = decltype(c)::value;
          constexpr int S = P::template slot_of<E, C>();
          const u32 v = __shfl_sync(0xffffffffu, get_e<P::W, S>(r), int(sl));
          res = (u32(C) == ct) ? v : res;
        });
        set_e<P::W, E>(o, res);
      });
    }
    if constexpr (P::TMA_STORE) {
      // outputs into this thread's own slots of the stage's src tile (read only by this
      // thread: the shuffle gather keeps sources in registers, the smem gather reads
      // its own staging area), then one cp.async.bulk of the contiguous dst tile
      const u32 ts = sbase + (i % NS) * TBST;
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        sts_vec<P::W, P::VLD>(ts + u32((thr ^ LdOff<P, K>::value()) * P::W), &o[((K << P::VLD) * P::W) / 4]);
      });
      fence_proxy_async();
      __syncthreads();
      if (threadIdx.x == 0) {
        bulk_s2g(dst + tile_base<P, true>(t) * P::W, ts, TBS);
        bulk_commit();
      }
    } else {
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        store_vec<P::W, P::VLD, K, P::NW, P::ST_HINT>(o, dst + (eoff ^ LdOff<P, K>::value()) * P::W);
      });
    }
    if constexpr (P::TMA || P::GATHER_SMEM) __syncthreads();
  }
  if constexpr (P::TMA_STORE) {
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

// ------------------------------------------------------------------ reduce (a12)
// the reduction over the axis bits of the tile — register adds, shfl.bfly
// over lanes, shared memory over warps — run in the fixed order of reading R-reduce
// (DESIGN.md §3): one step per in-tile logical axis bit t = 0, 1, ..., K-1, each
// v <- v(t = 0) (op) v(t = 1) at whichever level of the kernel layout holds bit t.
// Zero-column (broadcast) bits are skipped and de-duplicated at store.
// The reduction operator (ll_plan_opts.reduce_op): fp32 round-to-nearest add (no FMA
// contraction), max or min (exact: the result is one of the operands).
template <int OP> __device__ __forceinline__ float red_op(float a, float b) {
  if constexpr (OP == 1) return fmaxf(a, b);
  else if constexpr (OP == 2) return fminf(a, b);
  else return __fadd_rn(a, b);
}

template <class P, int S> struct RedStep {
  static constexpr int HB = P::AXIS_HW[S];
  static constexpr bool HREG = HB < P::R;
  static constexpr bool HWARP = HB >= P::R + 5;
  // registers no longer live at step S: reduced by an earlier register step, or duplicate
  static constexpr int dead() {
    int m = P::DUP_REG_MASK;
    for (int q = 0; q < S; ++q) if (P::AXIS_HW[q] < P::R) m |= 1 << P::AXIS_HW[q];
    return m;
  }
  // index of live register E among the live ones (the warp step's smem slot)
  template <int E> static constexpr int live_index() {
    int k = 0, t = 0;
    for (int b = 0; b < P::R; ++b) { if ((dead() >> b) & 1) continue; if ((E >> b) & 1) k |= 1 << t; ++t; }
    return k;
  }
};

template <class P>
__device__ __forceinline__ void ll_reduce_tile(u32 (&r)[1 << P::R], float* sm, u32 lane, u32 warp, u64 oblk,
                                               u64 othr, bool do_store, float* __restrict__ dst) {
  static_for<P::KB>([&](auto s) {
    using St = RedStep<P, decltype(s)::value>;
    constexpr int HB = St::HB;
    constexpr int DEAD = St::dead();
    if constexpr (St::HREG) {
      // register step: slot E (bit HB clear) takes r[E] (op) r[E | bit HB]
      static_for<(1 << P::R)>([&](auto e) {
        constexpr int E = decltype(e)::value;
        if constexpr (((E >> HB) & 1) == 0 && (E & DEAD) == 0)
          r[E] = __float_as_uint(red_op<P::OP>(__uint_as_float(r[E]), __uint_as_float(r[E | (1 << HB)])));
      });
    } else if constexpr (!St::HWARP) {
      // lane step: butterfly partner lane ^ bit; the lane with the bit clear computes
      // v(t = 0) (op) v(t = 1) — it is the copy later steps and the store use
      constexpr int LB = HB - P::R;
      static_for<(1 << P::R)>([&](auto e) {
        constexpr int E = decltype(e)::value;
        if constexpr ((E & DEAD) == 0) {
          const float x = __uint_as_float(r[E]);
          r[E] = __float_as_uint(red_op<P::OP>(x, __shfl_xor_sync(0xffffffffu, x, 1 << LB)));
        }
      });
    } else {
      // warp step through shared memory: [live slot][thread], partner warp ^ bit
      constexpr int WBIT = HB - P::R - 5;
      constexpr u32 NT = 32u << P::WB;
      static_for<(1 << P::R)>([&](auto e) {
        constexpr int E = decltype(e)::value;
        if constexpr ((E & DEAD) == 0)
          sm[St::template live_index<E>() * NT + threadIdx.x] = __uint_as_float(r[E]);
      });
      __syncthreads();
      const u32 pt = threadIdx.x ^ (32u << WBIT);
      static_for<(1 << P::R)>([&](auto e) {
        constexpr int E = decltype(e)::value;
        if constexpr ((E & DEAD) == 0)
          r[E] = __float_as_uint(red_op<P::OP>(__uint_as_float(r[E]), sm[St::template live_index<E>() * NT + pt]));
      });
      __syncthreads();
    }
    (void)warp;
  });
  if (do_store) {
    static_for<(1 << P::R)>([&](auto e) {
      constexpr int E = decltype(e)::value;
      if constexpr ((E & (P::RED_REG_MASK | P::DUP_REG_MASK)) == 0) {
        constexpr u64 oc = P::template out_of_slot<E>();
        dst[oblk ^ othr ^ oc] = __uint_as_float(r[E]);
      }
    });
  }
}

template <class P>
__device__ __forceinline__ void ll_reduce_body(const float* __restrict__ src, float* __restrict__ dst, u64 ntiles) {
  extern __shared__ __align__(16) u8 ll_smem[];
  ll_pdl_begin();
  const u32 lane = threadIdx.x & 31u;
  const u32 warp = threadIdx.x >> 5;
  u64 othr = 0;
  static_for<5>([&](auto t) {
    constexpr int T = decltype(t)::value;
    if ((lane >> T) & 1) othr ^= P::OUT_COL[P::R + T];
  });
  static_for<P::WB>([&](auto t) {
    constexpr int T = decltype(t)::value;
    if ((warp >> T) & 1) othr ^= P::OUT_COL[P::R + 5 + T];
  });
  const bool do_store = ((lane & P::NOSTORE_LANE_MASK) == 0) && ((warp & P::NOSTORE_WARP_MASK) == 0);
  auto out_blk = [&](u64 t) {
    u64 oblk = 0;
    static_for<P::G>([&](auto g) {
      constexpr int Gi = decltype(g)::value;
      if ((t >> Gi) & 1) oblk ^= P::GRID_OUT[Gi];
    });
    return oblk;
  };
  const u64 thr = thread_base<P, true>(lane, warp);
  if constexpr (P::TMA) {
    // The CTA tile of L is contiguous in HBM: one cp.async.bulk per tile into a
    // double-buffered stage, completion on an mbarrier; the next tile's copy is in
    // flight while this one is reduced.  Stage reads use the line-coalesced σ offsets
    // (16-byte vectors, 8 lanes per 128-byte row: conflict-free).
    constexpr u32 TB = u32(4) << (P::R + 5 + P::WB);
    constexpr u32 NS = P::STAGES;
    const u32 sbase = u32(__cvta_generic_to_shared(ll_smem));
    const u32 bar0 = sbase + NS * TB + P::WRED_BYTES;
    float* sm = reinterpret_cast<float*>(ll_smem + NS * TB);
    if (threadIdx.x == 0) {
      for (u32 q = 0; q < NS; ++q) mbar_init(bar0 + 8 * q, 1);
      mbar_fence_init();
    }
    __syncthreads();
    // prologue: the first NS - 1 tiles of this CTA are in flight before any compute
    if (threadIdx.x == 0) {
      for (u32 q = 0; q + 1 < NS; ++q) {
        const u64 tq = blockIdx.x + u64(q) * gridDim.x;
        if (tq < ntiles) {
          mbar_expect_tx(bar0 + 8 * q, TB);
          bulk_g2s(sbase + q * TB, reinterpret_cast<const u8*>(src) + tile_base<P, true>(tq), TB, bar0 + 8 * q);
        }
      }
    }
    u32 i = 0;
    for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
      const u32 st = i % NS;
      // refill the stage consumed in the previous iteration with tile i + NS - 1
      const u64 tn = t + u64(NS - 1) * gridDim.x;
      if (threadIdx.x == 0 && tn < ntiles) {
        const u32 sn = (i + NS - 1) % NS;
        fence_proxy_async();
        mbar_expect_tx(bar0 + 8 * sn, TB);
        bulk_g2s(sbase + sn * TB, reinterpret_cast<const u8*>(src) + tile_base<P, true>(tn), TB, bar0 + 8 * sn);
      }
      mbar_wait(bar0 + 8 * st, (i / NS) & 1u);
      u32 r[1 << P::R];
      const u32 tb = sbase + st * TB + u32(thr);
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        constexpr int E0 = K << P::VLD;
        lds_v4(tb + u32(LdOff<P, K>::value()), r[E0], r[E0 + 1], r[E0 + 2], r[E0 + 3]);
      });
      ll_reduce_tile<P>(r, sm, lane, warp, out_blk(t), othr, do_store, dst);
      __syncthreads();   // stage st is free before it is refilled next iteration
    }
  } else {
    float* sm = reinterpret_cast<float*>(ll_smem);
    for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const u8* s = reinterpret_cast<const u8*>(src) + (tile_base<P, true>(t) ^ thr);
      u32 r[1 << P::R];
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        load_vec<4, P::VLD, K, (1 << P::R), P::LD_L1>(r, s + LdOff<P, K>::value());
      });
      ll_reduce_tile<P>(r, sm, lane, warp, out_blk(t), othr, do_store, dst);
    }
  }
}

// ------------------------------------------------------------------ scan (N3)
// P:308 / SURVEY §8(f) N3: inclusive fp32 prefix sum along the axis inside each tile,
// in the fixed order of reading R-scan: for logical axis bit S = 0, 1,
// ..., an element whose bit S is set adds the value (before this step) of the last
// element of the lower half of its aligned 2^(S+1)-block — the position with the
// hardware bit of S cleared and the hardware bits of the lower axis bits set.  Those
// partner positions have bit S clear, so no step overwrites a value it still reads.
template <class P, int S> struct ScanStep {
  static constexpr int HB = P::AXIS_HW[S];
  static constexpr bool HREG = HB < P::R;
  static constexpr bool HWARP = HB >= P::R + 5;
  static constexpr u32 low_reg() { u32 m = 0; for (int q = 0; q < S; ++q) if (P::AXIS_HW[q] < P::R) m |= 1u << P::AXIS_HW[q]; return m; }
  static constexpr u32 low_lane() {
    u32 m = 0;
    for (int q = 0; q < S; ++q)
      if (P::AXIS_HW[q] >= P::R && P::AXIS_HW[q] < P::R + 5) m |= 1u << (P::AXIS_HW[q] - P::R);
    return m;
  }
  static constexpr u32 low_warp() { u32 m = 0; for (int q = 0; q < S; ++q) if (P::AXIS_HW[q] >= P::R + 5) m |= 1u << (P::AXIS_HW[q] - P::R - 5); return m; }
  static constexpr bool SMEM = HWARP || low_warp() != 0;
  static constexpr bool SHFL = !SMEM && (!HREG || low_lane() != 0);
};

// sm: NW x threads floats (the warp-crossing steps' exchange buffer)
template <class P>
__device__ __forceinline__ void ll_scan_steps(u32 (&r)[P::NW], u32 lane, float* sm) {
    static_for<P::KB>([&](auto s) {
      using St = ScanStep<P, decltype(s)::value>;
      constexpr int HB = St::HB;
      constexpr u32 LR = St::low_reg(), LL = St::low_lane();
      if constexpr (St::SMEM) {
        // bit S or a lower axis bit on the warps: every value goes through shared memory
        // ([slot][thread]); the partner is (slot, lane, warp) with the bit of S cleared
        // and the lower axis bits set
        constexpr u32 NT = 32u << P::WB;
        constexpr u32 LW = St::low_warp();
        const u32 warp = threadIdx.x >> 5;
        static_for<P::NW>([&](auto e) {
          constexpr int E = decltype(e)::value;
          sm[E * NT + threadIdx.x] = __uint_as_float(r[E]);
        });
        __syncthreads();
        u32 pl = lane | LL, pw = warp | LW;
        bool upper = true;
        if constexpr (St::HWARP) {
          constexpr int WBIT = HB - P::R - 5;
          pw &= ~(1u << WBIT);
          upper = (warp >> WBIT) & 1u;
        } else if constexpr (!St::HREG) {
          constexpr int LBIT = HB - P::R;
          pl &= ~(1u << LBIT);
          upper = (lane >> LBIT) & 1u;
        }
        const u32 pt = pw * 32u + pl;
        static_for<P::NW>([&](auto e) {
          constexpr int E = decltype(e)::value;
          if constexpr (!St::HREG || ((E >> HB) & 1)) {
            constexpr int E2 = (St::HREG ? (E & ~(1 << HB)) : E) | int(LR);
            if (upper) r[E] = __float_as_uint(red_op<P::OP>(__uint_as_float(r[E]), sm[E2 * NT + pt]));
          }
        });
        __syncthreads();
      } else if constexpr (!St::SHFL) {
        // bit S and every lower axis bit live in this thread's registers
        static_for<P::NW>([&](auto e) {
          constexpr int E = decltype(e)::value;
          if constexpr ((E >> HB) & 1) {
            constexpr int E2 = (E & ~(1 << HB)) | int(LR);
            r[E] = __float_as_uint(red_op<P::OP>(__uint_as_float(r[E]), __uint_as_float(r[E2])));
          }
        });
      } else if constexpr (St::HREG) {
        // bit S in registers, some lower axis bit in lanes: shuffle from lane | LL
        const int sl = int(lane | LL);
        static_for<P::NW>([&](auto e) {
          constexpr int E = decltype(e)::value;
          if constexpr ((E >> HB) & 1) {
            constexpr int E2 = (E & ~(1 << HB)) | int(LR);
            const float x = __shfl_sync(0xffffffffu, __uint_as_float(r[E2]), sl);
            r[E] = __float_as_uint(red_op<P::OP>(__uint_as_float(r[E]), x));
          }
        });
      } else {
        // bit S is a lane bit: every slot shuffles; the upper lanes add
        constexpr int LB = HB - P::R;
        const int sl = int((lane & ~(1u << LB)) | LL);
        const bool upper = (lane >> LB) & 1u;
        static_for<P::NW>([&](auto e) {
          constexpr int E = decltype(e)::value;
          constexpr int E2 = E | int(LR);
          const float x = __shfl_sync(0xffffffffu, __uint_as_float(r[E2]), sl);
          if (upper) r[E] = __float_as_uint(red_op<P::OP>(__uint_as_float(r[E]), x));
        });
      }
    });
}

template <class P>
__device__ __forceinline__ void ll_scan_body(const u8* __restrict__ src, u8* __restrict__ dst, u64 ntiles) {
  extern __shared__ __align__(16) u8 ll_smem[];
  ll_pdl_begin();
  const u32 lane = threadIdx.x & 31u;
  const u32 warp = threadIdx.x >> 5;
  const u64 thr = thread_base<P, true>(lane, warp);
  auto store_tile = [&](const u32 (&r)[P::NW], u64 base) {
    static_for<(1 << (P::R - P::VLD))>([&](auto k) {
      constexpr int K = decltype(k)::value;
      store_vec<4, P::VLD, K, P::NW, P::ST_HINT>(r, dst + base + LdOff<P, K>::value());
    });
  };
  if constexpr (P::TMA) {
    // the CTA tile is contiguous in HBM: cp.async.bulk into NS stages (mbarrier
    // completion, the next tiles in flight while this one is scanned), 16-byte stage
    // reads through the line σ, results stored from registers
    constexpr u32 TB = u32(4) << (P::R + 5 + P::WB);
    constexpr u32 NS = P::STAGES;
    const u32 sbase = u32(__cvta_generic_to_shared(ll_smem));
    const u32 bar0 = sbase + NS * TB + P::XS_BYTES;
    float* xs = reinterpret_cast<float*>(ll_smem + NS * TB);
    if (threadIdx.x == 0) {
      for (u32 q = 0; q < NS; ++q) mbar_init(bar0 + 8 * q, 1);
      mbar_fence_init();
    }
    __syncthreads();
    auto issue = [&](u64 tq, u32 q) {
      mbar_expect_tx(bar0 + 8 * q, TB);
      bulk_g2s(sbase + q * TB, src + tile_base<P, true>(tq), TB, bar0 + 8 * q);
    };
    if (threadIdx.x == 0)
      for (u32 q = 0; q + 1 < NS; ++q)
        if (blockIdx.x + u64(q) * gridDim.x < ntiles) issue(blockIdx.x + u64(q) * gridDim.x, q);
    u32 i = 0;
    for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
      const u32 st = i % NS;
      const u64 tn = t + u64(NS - 1) * gridDim.x;
      if constexpr (!P::TMA_STORE) {
        if (threadIdx.x == 0 && tn < ntiles) {
          fence_proxy_async();
          issue(tn, (i + NS - 1) % NS);
        }
      }
      mbar_wait(bar0 + 8 * st, (i / NS) & 1u);
      u32 r[P::NW];
      const u32 tb = sbase + st * TB + u32(thr);
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        constexpr int E0 = K << P::VLD;
        lds_v4(tb + u32(LdOff<P, K>::value()), r[E0], r[E0 + 1], r[E0 + 2], r[E0 + 3]);
      });
      if constexpr (!P::TMA_STORE) __syncthreads();   // stage st read by every thread before it is refilled
      ll_scan_steps<P>(r, lane, xs);
      if constexpr (P::TMA_STORE) {
        // results back into this thread's own 16-byte slots of the stage, then one
        // cp.async.bulk shared -> global of the whole (contiguous) dst tile
        static_for<(1 << (P::R - P::VLD))>([&](auto k) {
          constexpr int K = decltype(k)::value;
          constexpr int E0 = K << P::VLD;
          sts_vec<4, 2>(tb + u32(LdOff<P, K>::value()), &r[E0]);
        });
        fence_proxy_async();
        __syncthreads();
        if (threadIdx.x == 0) {
          bulk_s2g(dst + tile_base<P, true>(t), sbase + st * TB, TB);
          bulk_commit();
          // refill the stage of the PREVIOUS tile (its bulk store has had this whole
          // iteration to read it out: allow only this tile's store to be pending) with
          // tile i + NS - 1 — the loads stay NS - 1 tiles ahead without waiting on the
          // store just issued
          if (tn < ntiles) {
            bulk_wait_read<1>();
            fence_proxy_async();
            issue(tn, (i + NS - 1) % NS);
          }
        }
      } else {
        store_tile(r, tile_base<P, true>(t) ^ thr);
      }
    }
    if constexpr (P::TMA_STORE) {
      if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
  } else {
    float* xs = reinterpret_cast<float*>(ll_smem);
    for (u64 t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const u64 base = tile_base<P, true>(t) ^ thr;
      u32 r[P::NW];
      static_for<(1 << (P::R - P::VLD))>([&](auto k) {
        constexpr int K = decltype(k)::value;
        load_vec<4, P::VLD, K, P::NW, P::LD_L1>(r, src + base + LdOff<P, K>::value());
      });
      ll_scan_steps<P>(r, lane, xs);
      store_tile(r, base);
    }
  }
}
