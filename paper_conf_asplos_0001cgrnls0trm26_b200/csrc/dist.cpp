// DEVICE-class plans (row a9; north star): a layout whose F2 matrix maps bits to a
// device dimension, converted to one that maps different bits to it.  The pull map Q
// crosses devices; the plan decomposes it into
//   pack      — a local conversion A_local -> S (send layout: the receiver's rank bits
//               on top, each peer's chunk contiguous and in the receiver's order),
//   exchange  — one all-to-all of equal chunks over NVLink (grouped ncclSend/ncclRecv),
//   unpack    — a local conversion R -> B_local (R: the source rank bits on top);
// both local stages are ordinary plans (CTA / SMEM class tile kernels, or NOOP).
// NCCL is loaded with dlopen (libnccl.so.2: the one torch already loaded, else the
// system one; LL_NCCL_LIB overrides).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cstring>
#include <map>
#include <mutex>

#include "ll_internal.hpp"

namespace ll {
ll_status convert_impl(const void* src, void* dst, void* ws, ConvPlan& P, cudaStream_t st);

namespace {

struct NcclUid { char internal[128]; };
struct Nccl {
  void* h = nullptr;
  int (*getUniqueId)(NcclUid*) = nullptr;
  int (*commInitRank)(void**, int, NcclUid, int) = nullptr;
  int (*commDestroy)(void*) = nullptr;
  int (*groupStart)() = nullptr;
  int (*groupEnd)() = nullptr;
  int (*send)(const void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*recv)(void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  const char* (*errstr)(int) = nullptr;
  int (*asyncError)(void*, int*) = nullptr;
};

Nccl& nccl() {
  static Nccl n;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* env = getenv("LL_NCCL_LIB");
    const char* names[] = {env && *env ? env : "libnccl.so.2", "libnccl.so"};
    for (const char* nm : names) {
      n.h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
      if (n.h) break;
    }
    if (!n.h) return;
    n.getUniqueId = reinterpret_cast<decltype(n.getUniqueId)>(dlsym(n.h, "ncclGetUniqueId"));
    n.commInitRank = reinterpret_cast<decltype(n.commInitRank)>(dlsym(n.h, "ncclCommInitRank"));
    n.commDestroy = reinterpret_cast<decltype(n.commDestroy)>(dlsym(n.h, "ncclCommDestroy"));
    n.groupStart = reinterpret_cast<decltype(n.groupStart)>(dlsym(n.h, "ncclGroupStart"));
    n.groupEnd = reinterpret_cast<decltype(n.groupEnd)>(dlsym(n.h, "ncclGroupEnd"));
    n.send = reinterpret_cast<decltype(n.send)>(dlsym(n.h, "ncclSend"));
    n.recv = reinterpret_cast<decltype(n.recv)>(dlsym(n.h, "ncclRecv"));
    n.errstr = reinterpret_cast<decltype(n.errstr)>(dlsym(n.h, "ncclGetErrorString"));
    n.asyncError = reinterpret_cast<decltype(n.asyncError)>(dlsym(n.h, "ncclCommGetAsyncError"));
  });
  if (!n.h || !n.send || !n.recv || !n.commInitRank) fail(LL_ERR_NCCL, "libnccl.so.2 not available");
  return n;
}

// CUDA IPC mappings opened in this process (one per exported block).
struct IpcMap { void* base; int refs; };
struct IpcRegistry {
  std::mutex mu;
  std::map<std::string, IpcMap> by_handle;
  std::vector<std::pair<void*, std::string>> mapped;
};
IpcRegistry& ipc_registry() {
  static IpcRegistry r;
  return r;
}

// Base and size of the allocation containing p (driver cuMemGetAddressRange through
// the runtime's entry-point table; the library links only cudart).
cudaError_t mem_range(const void* p, void** base, size_t* size) {
  typedef int (*Fn)(unsigned long long*, size_t*, unsigned long long);
  static Fn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t e = cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q);
    if (e != cudaSuccess) return e;
    if (!f || q != cudaDriverEntryPointSuccess) return cudaErrorNotSupported;
    fn = reinterpret_cast<Fn>(f);
  }
  unsigned long long b = 0;
  int r = fn(&b, size, reinterpret_cast<unsigned long long>(p));
  if (r != 0) return cudaErrorInvalidValue;
  *base = reinterpret_cast<void*>(b);
  return cudaSuccess;
}

void check_nccl(int r, const char* what) {
  if (r != 0) fail(LL_ERR_NCCL, std::string(what) + ": " + (nccl().errstr ? nccl().errstr(r) : "error"));
}

// Relabel two layouts with the same set of unit columns onto a compact logical space
// ("x", n bits) numbered by L1's column order: conversion depends only on how the
// two layouts relate, and the local slices cover only part of the logical tensor.
void relabel(const Layout& L1, const Layout& L2, Layout& R1, Layout& R2) {
  const int n = int(L1.cols.size());
  auto idx = [&](u64 c) {
    for (int k = 0; k < n; ++k) if (L1.cols[k] == c) return k;
    fail(LL_ERR_UNSUPPORTED, "device plan: local column sets differ (internal)");
  };
  R1.in = L1.in; R2.in = L2.in;
  R1.out = R2.out = {Dim{"x", n}};
  R1.cols.clear(); R2.cols.clear();
  for (int k = 0; k < n; ++k) R1.cols.push_back(u64(1) << k);
  for (u64 c : L2.cols) R2.cols.push_back(u64(1) << idx(c));
}

Layout local_of(const Layout& L) {
  Layout R;
  for (auto& d : L.in) if (d.name != "dev" && d.name != "device") R.in.push_back(d);
  R.out = L.out;
  int n = 0;
  for (auto& d : R.in) n += d.bits;
  R.cols.assign(L.cols.begin(), L.cols.begin() + n);
  return R;
}

Layout memory_layout(const std::vector<u64>& cols, const std::vector<Dim>& out) {
  Layout R;
  R.in = {Dim{"offset", int(cols.size())}};
  R.out = out;
  R.cols = cols;
  return R;
}

}  // namespace

// §8(f) N4: the DEVICE map as ONE tile kernel per rank.  The pair (A, B) is planned
// over the GLOBAL packed index space (local bits, then the dev bits on top: the
// layouts read as memory layouts of 2^{d_in} elements), which gives an ordinary CTA
// tile plan.  Push form: every tile's loads must be rank-local, so the src dev bits
// are grid bits; they are moved to the top of the CTA index, and rank r runs the
// 2^{G-p} tiles above r * 2^{G-p}.  Its stores land in the receivers' windows through
// the global dst offset's top bits (DstPeers in ll_kernels.cuh): no pack, exchange
// buffer or unpack pass, and the NVLink transfer overlaps the loads tile by tile.
void plan_peer(ConvPlan& P, const ll_plan_opts* opts) {
  const Layout &A = P.A, &B = P.B;
  const int p = A.in_bits("dev");
  const int nloc = A.d_in() - p;
  if (A.in_pos("dev") != nloc || B.in_pos("dev") != B.d_in() - p)
    fail(LL_ERR_UNSUPPORTED, "peer exchange: the dev dimension must be declared last");
  ll_plan_opts lo;
  std::memset(&lo, 0, sizeof lo);
  lo.force_class = -1;
  lo.max_vec_bytes = opts->max_vec_bytes ? opts->max_vec_bytes : 16;
  lo.tile_bytes = opts->tile_bytes;
  lo.thread_bytes = opts->thread_bytes;
  // 8-byte elements move as pairs of 4-byte atoms (one more, lowest, local bit)
  Layout Ag = memory_layout(A.cols, A.out), Bg = memory_layout(B.cols, B.out);
  int wk = P.w, nl = nloc;
  if (P.w == 8) { Ag = atomize(Ag); Bg = atomize(Bg); wk = 4; nl = nloc + 1; }
  u64 devmask = 0;
  for (int t = 0; t < p; ++t) devmask |= u64(1) << (nl + t);
  auto F = plan_convert(Ag, Bg, wk, &lo, devmask);
  if (F->exec != EXEC_TILE || !F->tile.ld_xcol.empty() || !F->tile.rep_bits.empty())
    fail(LL_ERR_UNSUPPORTED, "peer exchange: the global map has no permutation tile plan");
  TilePlan& T = F->tile;
  for (int b : T.ld_bit)
    if (b >= nl) fail(LL_ERR_UNSUPPORTED, "peer exchange: a src tile spans ranks (use the collective exchange)");
  std::vector<int> gs, gd;
  std::vector<std::pair<int, int>> hi;
  for (size_t g = 0; g < T.grid_src_bit.size(); ++g) {
    if (T.grid_src_bit[g] >= nl) hi.push_back({T.grid_src_bit[g], T.grid_dst_bit[g]});
    else { gs.push_back(T.grid_src_bit[g]); gd.push_back(T.grid_dst_bit[g]); }
  }
  if (int(hi.size()) != p) fail(LL_ERR_UNSUPPORTED, "peer exchange: src dev bits are not grid bits (internal)");
  std::sort(hi.begin(), hi.end());
  for (auto& h : hi) { gs.push_back(h.first); gd.push_back(h.second); }
  T.grid_src_bit = gs;
  T.grid_dst_bit = gd;
  F->peer_shift = nl;
  F->peer_reg = false;
  for (int b = 0; b < T.R; ++b)
    if (T.st_bit[b] >= nl) F->peer_reg = true;
  F->source = codegen_tile(*F);
  P.rank_tiles = u64(1) << (gs.size() - p);
  P.fused = std::move(F);
  P.exchange = LL_EXCHANGE_PEER;
  P.nranks = opts->comm->nranks;
  P.comm = opts->comm;
  P.local_elems = u64(1) << nloc;
  P.chunk_elems = u64(1) << (nloc - p);
  P.workspace_bytes = 0;
  P.src_elems = P.dst_elems = P.local_elems;
}

void plan_device(ConvPlan& P, const ll_plan_opts* opts) {
  if (!opts || !opts->comm) fail(LL_ERR_INVALID_ARG, "DEVICE plans require opts->comm (the map mixes device bits)");
  {
    const int p = P.A.in_bits("dev");
    if (P.B.in_bits("dev") != p || p == 0) fail(LL_ERR_UNSUPPORTED, "DEVICE: A and B need the same number of dev bits");
    if (!P.A.unit_columns() || !P.B.unit_columns())
      fail(LL_ERR_UNSUPPORTED, "DEVICE: only bijective permutation layouts are supported");
    if (opts->comm->nranks != (1 << p)) fail(LL_ERR_INVALID_ARG, "DEVICE: communicator size != 2^(dev bits)");
    const bool windows = !opts->comm->peer_dst.empty();
    int ex = opts->exchange;
    if (ex == LL_EXCHANGE_AUTO) ex = windows ? LL_EXCHANGE_PEER : LL_EXCHANGE_COLLECTIVE;
    if (ex == LL_EXCHANGE_PEER) {
      if (!windows && !opts->comm->loopback)
        fail(LL_ERR_INVALID_ARG, "peer exchange needs a communicator with peer windows (ll_comm_create_peers)");
      plan_peer(P, opts);
      return;
    }
    if (!opts->comm->nccl && !opts->comm->loopback)
      fail(LL_ERR_INVALID_ARG, "collective exchange needs an NCCL (or loopback) communicator");
  }
  const Layout &A = P.A, &B = P.B;
  const int p = A.in_bits("dev");
  if (B.in_bits("dev") != p || p == 0) fail(LL_ERR_UNSUPPORTED, "DEVICE: A and B need the same number of dev bits");
  if (!A.unit_columns() || !B.unit_columns())
    fail(LL_ERR_UNSUPPORTED, "DEVICE: only bijective permutation layouts are supported");
  ll_comm* comm = opts->comm;
  if (comm->nranks != (1 << p)) fail(LL_ERR_INVALID_ARG, "DEVICE: communicator size != 2^(dev bits)");
  Layout Al = local_of(A), Bl = local_of(B);
  const int nloc = Al.d_in();
  const int pa = A.in_pos("dev"), pb = B.in_pos("dev");
  std::vector<u64> a(p), b(p);
  for (int t = 0; t < p; ++t) { a[t] = A.cols[pa + t]; b[t] = B.cols[pb + t]; }
  auto in = [](const std::vector<u64>& v, u64 c) { return std::find(v.begin(), v.end(), c) != v.end(); };
  // Logical bits by where they live: LL (local in both), LD (A-local, B-dev: they pick
  // the receiver), DL (A-dev, B-local: they pick the sender), DD (a dev bit of both: the
  // rank bit is fixed or relabelled, SURVEY §8(e)(2) partial exchange).  Rank r sends
  // 2^xk chunks (xk = |LD| = |DL|) to the ranks whose B-dev coordinates agree with r on
  // the DD columns, and receives 2^xk chunks from the ranks whose A-dev coordinates agree
  // with r's B-dev coordinates there; all chunks are equal (bijective layouts).
  std::vector<u64> LD, DL;
  for (int t = 0; t < p; ++t) if (in(Al.cols, b[t])) LD.push_back(b[t]);   // B-dev order
  for (int t = 0; t < p; ++t) if (in(Bl.cols, a[t])) DL.push_back(a[t]);   // A-dev order
  if (LD.size() != DL.size()) fail(LL_ERR_UNSUPPORTED, "DEVICE: unequal send / receive bits (internal)");
  const int xk = int(LD.size());
  P.xk = xk;
  P.send_jcol.assign(xk, 0);
  P.send_rcol.assign(p, 0);
  P.recv_icol.assign(xk, 0);
  P.recv_rcol.assign(p, 0);
  {
    int j = 0;
    for (int t = 0; t < p; ++t) {
      if (in(Al.cols, b[t])) { P.send_jcol[j++] = 1u << t; continue; }
      // DD: receiver's B-dev bit t = sender's A-dev bit t' with the same column
      for (int t2 = 0; t2 < p; ++t2) if (a[t2] == b[t]) P.send_rcol[t2] ^= 1u << t;
    }
    int i = 0;
    for (int t = 0; t < p; ++t) {
      if (in(Bl.cols, a[t])) { P.recv_icol[i++] = 1u << t; continue; }
      // DD: sender's A-dev bit t = receiver's B-dev bit t' with the same column
      for (int t2 = 0; t2 < p; ++t2) if (b[t2] == a[t]) P.recv_rcol[t2] ^= 1u << t;
    }
  }
  // C: B-local vectors that are A-local too (LL), in B's order
  std::vector<u64> C;
  for (u64 c : Bl.cols) if (!in(a, c)) C.push_back(c);
  std::vector<u64> scols = C, rcols = C;
  scols.insert(scols.end(), LD.begin(), LD.end());   // send: chunk (receiver) bits on top
  rcols.insert(rcols.end(), DL.begin(), DL.end());   // recv: chunk (sender) bits on top
  Layout S = memory_layout(scols, A.out), R = memory_layout(rcols, A.out);
  ll_plan_opts lo;
  std::memset(&lo, 0, sizeof lo);
  lo.force_class = -1;
  lo.max_vec_bytes = opts->max_vec_bytes ? opts->max_vec_bytes : 16;
  lo.tile_bytes = opts->tile_bytes;
  lo.thread_bytes = opts->thread_bytes;
  Layout A1, S1, R1, B1;
  relabel(Al, S, A1, S1);
  relabel(R, Bl, R1, B1);
  int wk = P.w;
  if (P.w == 8) { A1 = atomize(A1); S1 = atomize(S1); R1 = atomize(R1); B1 = atomize(B1); wk = 4; }
  auto pack = plan_convert(A1, S1, wk, &lo);
  auto unpack = plan_convert(R1, B1, wk, &lo);
  P.pack = pack->exec == EXEC_NOOP ? nullptr : std::move(pack);
  P.unpack = unpack->exec == EXEC_NOOP ? nullptr : std::move(unpack);
  P.nranks = comm->nranks;
  P.comm = comm;
  P.local_elems = u64(1) << nloc;
  P.chunk_elems = u64(1) << (nloc - xk);
  const size_t lb = size_t(P.local_elems) * P.w;
  const size_t per_rank = (P.pack ? lb : 0) + (P.unpack ? lb : 0);
  P.workspace_bytes = comm->loopback ? per_rank * comm->nranks : per_rank;
  P.src_elems = P.dst_elems = P.local_elems;
}

void ensure_tile_kernel(ConvPlan& P);
unsigned grid_for_tiles(u64 ntiles);
int launch_peer_barrier(void* const* flags, int nranks, int rank, unsigned epoch, cudaStream_t st);

namespace {
void launch_peer_tiles(ConvPlan& F, const void* src, const LLPeersHost& tab, u64 ntiles, u64 tile0, cudaStream_t st) {
  unsigned long long nt = ntiles, t0 = tile0;
  void* args[] = {const_cast<void**>(&src), const_cast<LLPeersHost*>(&tab), &nt, &t0};
  launch_kernel(F.kernel, grid_for_tiles(ntiles), F.tile.threads(), args, size_t(F.smem_bytes), st,
                "cudaLaunchKernelEx(ll_tile_peer_kernel)");
}
}  // namespace

ll_status peer_convert(ConvPlan& P, const void* src, void* dst, cudaStream_t st) {
  ll_comm* comm = P.comm;
  ConvPlan& F = *P.fused;
  ensure_tile_kernel(F);
  const size_t lb = size_t(P.local_elems) * P.w;
  LLPeersHost tab;
  std::memset(&tab, 0, sizeof tab);
  if (comm->loopback) {
    // virtual ranks in one buffer: the windows are the slices.  Rank r's tiles are the
    // CTA indices [r * rank_tiles, (r + 1) * rank_tiles) of the global plan and its src
    // slice starts at r * lb, i.e. all ranks together are exactly one launch over every
    // tile with src = the whole buffer (no per-rank ramp and tail)
    for (int q = 0; q < P.nranks; ++q) tab.dst[q] = static_cast<char*>(dst) + q * lb;
    launch_peer_tiles(F, src, tab, P.rank_tiles * u64(P.nranks), 0, st);
    return LL_OK;
  }
  if (dst != comm->peer_dst[comm->rank])
    fail(LL_ERR_INVALID_ARG, "peer exchange: dst must be this rank's registered window");
  if (comm->window_bytes < lb) fail(LL_ERR_INVALID_ARG, "peer exchange: window smaller than the local dst");
  for (int q = 0; q < P.nranks; ++q) tab.dst[q] = static_cast<char*>(comm->peer_dst[q]);
  // entry barrier: every receiver is done with its window's previous contents
  int e = launch_peer_barrier(comm->peer_flags.data(), P.nranks, comm->rank, ++comm->epoch, st);
  check_cuda(cudaError_t(e), "ll_peer_barrier_kernel");
  launch_peer_tiles(F, src, tab, P.rank_tiles, u64(comm->rank) * P.rank_tiles, st);
  // exit barrier: every sender's stores into this window have landed
  e = launch_peer_barrier(comm->peer_flags.data(), P.nranks, comm->rank, ++comm->epoch, st);
  check_cuda(cudaError_t(e), "ll_peer_barrier_kernel");
  return LL_OK;
}

ll_status device_convert(const ConvPlan& Pc, const void* src, void* dst, void* ws, cudaStream_t st) {
  ConvPlan& P = const_cast<ConvPlan&>(Pc);
  if (P.exchange == LL_EXCHANGE_PEER) return peer_convert(P, src, dst, st);
  ll_comm* comm = P.comm;
  const size_t lb = size_t(P.local_elems) * P.w, cb = size_t(P.chunk_elems) * P.w;
  if (P.workspace_bytes && !ws) fail(LL_ERR_INVALID_ARG, "DEVICE plan needs a workspace (ll_plan_workspace_bytes)");
  const int N = P.nranks;
  const int nloc_ranks = comm->loopback ? N : 1;
  const size_t per_rank = (P.pack ? lb : 0) + (P.unpack ? lb : 0);
  auto sendbuf = [&](int r) -> const char* {
    return P.pack ? static_cast<char*>(ws) + r * per_rank : static_cast<const char*>(src) + r * lb;
  };
  auto recvbuf = [&](int r) -> char* {
    return P.unpack ? static_cast<char*>(ws) + r * per_rank + (P.pack ? lb : 0) : static_cast<char*>(dst) + r * lb;
  };
  // 1. pack (local conversion on every local rank slice)
  if (P.pack)
    for (int r = 0; r < nloc_ranks; ++r)
      convert_impl(static_cast<const char*>(src) + r * lb, const_cast<char*>(sendbuf(r)), nullptr, *P.pack, st);
  // 2. exchange: send chunk j of rank s -> rank q = send_peer(j, s), which files it as
  // its recv chunk i with recv_peer(i, q) = s (all 2^xk chunks equal; grouped point-to-
  // point, so partial exchanges only talk to the ranks they share data with)
  const u64 nch = u64(1) << P.xk;
  if (comm->loopback) {
    for (int s = 0; s < N; ++s)
      for (u64 j = 0; j < nch; ++j) {
        const int q = P.send_peer(j, s);
        u64 i = 0;
        while (i < nch && P.recv_peer(i, q) != s) ++i;
        if (i == nch) fail(LL_ERR_UNSUPPORTED, "DEVICE: inconsistent chunk routing (internal)");
        cudaError_t e = cudaMemcpyAsync(recvbuf(q) + i * cb, sendbuf(s) + j * cb, cb, cudaMemcpyDeviceToDevice, st);
        if (e != cudaSuccess) fail(LL_ERR_CUDA, std::string("loopback exchange: ") + cudaGetErrorString(e));
      }
  } else {
    Nccl& n = nccl();
    check_nccl(n.groupStart(), "ncclGroupStart");
    for (u64 j = 0; j < nch; ++j)
      check_nccl(n.send(sendbuf(0) + j * cb, cb, /*ncclInt8*/ 0, P.send_peer(j, comm->rank), comm->nccl, st), "ncclSend");
    for (u64 i = 0; i < nch; ++i)
      check_nccl(n.recv(recvbuf(0) + i * cb, cb, 0, P.recv_peer(i, comm->rank), comm->nccl, st), "ncclRecv");
    check_nccl(n.groupEnd(), "ncclGroupEnd");
    // an earlier asynchronous NCCL failure on this communicator surfaces here
    int aerr = 0;
    if (n.asyncError) check_nccl(n.asyncError(comm->nccl, &aerr), "ncclCommGetAsyncError");
    check_nccl(aerr, "NCCL asynchronous error");
  }
  // 3. unpack
  if (P.unpack)
    for (int r = 0; r < nloc_ranks; ++r)
      convert_impl(recvbuf(r), static_cast<char*>(dst) + r * lb, nullptr, *P.unpack, st);
  return LL_OK;
}

}  // namespace ll

extern "C" {

ll_status ll_comm_get_unique_id(void* id) {
  try {
    if (!id) ll::fail(LL_ERR_INVALID_ARG, "null id");
    ll::NcclUid u;
    ll::check_nccl(ll::nccl().getUniqueId(&u), "ncclGetUniqueId");
    std::memcpy(id, &u, sizeof u);
    return LL_OK;
  } catch (const ll::Error& e) {
    ll::set_last_error(e.what());
    return e.st;
  }
}

ll_status ll_comm_create(const void* id, int nranks, int rank, ll_comm** out) {
  try {
    if (!id || !out || nranks < 1 || rank < 0 || rank >= nranks) ll::fail(LL_ERR_INVALID_ARG, "bad argument");
    auto c = std::make_unique<ll_comm>();
    c->nranks = nranks;
    c->rank = rank;
    ll::NcclUid u;
    std::memcpy(&u, id, sizeof u);
    ll::check_nccl(ll::nccl().commInitRank(&c->nccl, nranks, u, rank), "ncclCommInitRank");
    *out = c.release();
    return LL_OK;
  } catch (const ll::Error& e) {
    ll::set_last_error(e.what());
    return e.st;
  }
}

ll_status ll_comm_create_peers(int nranks, int rank, void* const* dst_windows, void* const* flag_bufs,
                               size_t window_bytes, ll_comm** out) {
  try {
    if (!out || !dst_windows || !flag_bufs || nranks < 1 || nranks > LL_MAX_PEERS || (nranks & (nranks - 1)) ||
        rank < 0 || rank >= nranks)
      ll::fail(LL_ERR_INVALID_ARG, "peer communicator: bad nranks / rank / buffers");
    auto c = std::make_unique<ll_comm>();
    c->nranks = nranks;
    c->rank = rank;
    c->window_bytes = window_bytes;
    for (int q = 0; q < nranks; ++q) {
      if (!dst_windows[q] || !flag_bufs[q]) ll::fail(LL_ERR_INVALID_ARG, "peer communicator: null window");
      if ((reinterpret_cast<uintptr_t>(dst_windows[q]) & 15) || (reinterpret_cast<uintptr_t>(flag_bufs[q]) & 15))
        ll::fail(LL_ERR_MISALIGNED, "peer communicator: windows must be 16-byte aligned");
      c->peer_dst.push_back(dst_windows[q]);
      c->peer_flags.push_back(flag_bufs[q]);
    }
    *out = c.release();
    return LL_OK;
  } catch (const ll::Error& e) {
    ll::set_last_error(e.what());
    return e.st;
  }
}

ll_status ll_ipc_export(const void* ptr, void* handle) {
  try {
    if (!ptr || !handle) ll::fail(LL_ERR_INVALID_ARG, "null argument");
    void* base = nullptr;
    size_t size = 0;
    ll::check_cuda(ll::mem_range(ptr, &base, &size), "cuMemGetAddressRange");
    cudaIpcMemHandle_t h;
    ll::check_cuda(cudaIpcGetMemHandle(&h, base), "cudaIpcGetMemHandle");
    uint64_t off = static_cast<const char*>(ptr) - static_cast<char*>(base);
    std::memcpy(handle, &h, sizeof h);
    std::memcpy(static_cast<char*>(handle) + 64, &off, 8);
    return LL_OK;
  } catch (const ll::Error& e) {
    ll::set_last_error(e.what());
    return e.st;
  }
}

ll_status ll_ipc_import(const void* handle, void** ptr) {
  try {
    if (!handle || !ptr) ll::fail(LL_ERR_INVALID_ARG, "null argument");
    std::string key(static_cast<const char*>(handle), 64);
    uint64_t off;
    std::memcpy(&off, static_cast<const char*>(handle) + 64, 8);
    auto& reg = ll::ipc_registry();
    std::lock_guard<std::mutex> g(reg.mu);
    auto it = reg.by_handle.find(key);
    if (it == reg.by_handle.end()) {
      cudaIpcMemHandle_t h;
      std::memcpy(&h, handle, sizeof h);
      void* base = nullptr;
      ll::check_cuda(cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
      it = reg.by_handle.emplace(key, ll::IpcMap{base, 0}).first;
    }
    it->second.refs += 1;
    *ptr = static_cast<char*>(it->second.base) + off;
    reg.mapped.push_back({*ptr, key});
    return LL_OK;
  } catch (const ll::Error& e) {
    ll::set_last_error(e.what());
    return e.st;
  }
}

ll_status ll_ipc_close(void* ptr) {
  try {
    auto& reg = ll::ipc_registry();
    std::lock_guard<std::mutex> g(reg.mu);
    for (size_t i = 0; i < reg.mapped.size(); ++i) {
      if (reg.mapped[i].first != ptr) continue;
      auto it = reg.by_handle.find(reg.mapped[i].second);
      reg.mapped.erase(reg.mapped.begin() + i);
      if (it != reg.by_handle.end() && --it->second.refs == 0) {
        cudaError_t e = cudaIpcCloseMemHandle(it->second.base);
        reg.by_handle.erase(it);
        ll::check_cuda(e, "cudaIpcCloseMemHandle");
      }
      return LL_OK;
    }
    ll::fail(LL_ERR_INVALID_ARG, "ll_ipc_close: pointer was not imported");
  } catch (const ll::Error& e) {
    ll::set_last_error(e.what());
    return e.st;
  }
  return LL_OK;
}

ll_status ll_comm_create_loopback(int nranks, ll_comm** out) {
  if (!out || nranks < 1 || (nranks & (nranks - 1))) {
    ll::set_last_error("loopback communicator: nranks must be a power of two");
    return LL_ERR_INVALID_ARG;
  }
  auto c = std::make_unique<ll_comm>();
  c->nranks = nranks;
  c->rank = -1;
  c->loopback = true;
  *out = c.release();
  return LL_OK;
}

ll_status ll_comm_check(const ll_comm* c) {
  try {
    if (!c) ll::fail(LL_ERR_INVALID_ARG, "null communicator");
    if (!c->nccl) return LL_OK;   // loopback / peer windows: errors surface as CUDA errors
    ll::Nccl& n = ll::nccl();
    if (!n.asyncError) ll::fail(LL_ERR_NCCL, "ncclCommGetAsyncError not available");
    int aerr = 0;
    ll::check_nccl(n.asyncError(c->nccl, &aerr), "ncclCommGetAsyncError");
    ll::check_nccl(aerr, "NCCL asynchronous error");
  } catch (const ll::Error& e) {
    ll::set_last_error(e.what());
    return e.st;
  }
  return LL_OK;
}

void ll_comm_destroy(ll_comm* c) {
  if (!c) return;
  if (c->nccl) {
    try { ll::nccl().commDestroy(c->nccl); } catch (...) {}
  }
  delete c;
}

}  // extern "C"
