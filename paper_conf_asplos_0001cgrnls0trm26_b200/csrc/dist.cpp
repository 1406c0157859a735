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
  });
  if (!n.h || !n.send || !n.recv || !n.commInitRank) fail(LL_ERR_NCCL, "libnccl.so.2 not available");
  return n;
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

void plan_device(ConvPlan& P, const ll_plan_opts* opts) {
  if (!opts || !opts->comm) fail(LL_ERR_INVALID_ARG, "DEVICE plans require opts->comm (the map mixes device bits)");
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
  for (int t = 0; t < p; ++t) {
    if (!in(Bl.cols, a[t]) || !in(Al.cols, b[t]))
      fail(LL_ERR_UNSUPPORTED, "DEVICE: partial device exchanges (dev bits shared by A and B) are not supported");
  }
  // C_B: B-local vectors that are A-local too, in B's order
  std::vector<u64> C;
  for (u64 c : Bl.cols) if (!in(a, c)) C.push_back(c);
  std::vector<u64> scols = C, rcols = C;
  scols.insert(scols.end(), b.begin(), b.end());   // send: receiver rank bits on top
  rcols.insert(rcols.end(), a.begin(), a.end());   // recv: source rank bits on top
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
  auto pack = plan_convert(A1, S1, P.w, &lo);
  auto unpack = plan_convert(R1, B1, P.w, &lo);
  P.pack = pack->exec == EXEC_NOOP ? nullptr : std::move(pack);
  P.unpack = unpack->exec == EXEC_NOOP ? nullptr : std::move(unpack);
  P.nranks = comm->nranks;
  P.comm = comm;
  P.local_elems = u64(1) << nloc;
  P.chunk_elems = u64(1) << (nloc - p);
  const size_t lb = size_t(P.local_elems) * P.w;
  const size_t per_rank = (P.pack ? lb : 0) + (P.unpack ? lb : 0);
  P.workspace_bytes = comm->loopback ? per_rank * comm->nranks : per_rank;
  P.src_elems = P.dst_elems = P.local_elems;
}

ll_status device_convert(const ConvPlan& Pc, const void* src, void* dst, void* ws, cudaStream_t st) {
  ConvPlan& P = const_cast<ConvPlan&>(Pc);
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
  // 2. exchange: chunk q of rank s's send buffer -> chunk s of rank q's recv buffer
  if (comm->loopback) {
    for (int s = 0; s < N; ++s)
      for (int q = 0; q < N; ++q) {
        cudaError_t e = cudaMemcpyAsync(recvbuf(q) + s * cb, sendbuf(s) + q * cb, cb, cudaMemcpyDeviceToDevice, st);
        if (e != cudaSuccess) fail(LL_ERR_CUDA, std::string("loopback exchange: ") + cudaGetErrorString(e));
      }
  } else {
    Nccl& n = nccl();
    check_nccl(n.groupStart(), "ncclGroupStart");
    for (int q = 0; q < N; ++q) {
      check_nccl(n.send(sendbuf(0) + q * cb, cb, /*ncclInt8*/ 0, q, comm->nccl, st), "ncclSend");
      check_nccl(n.recv(recvbuf(0) + q * cb, cb, 0, q, comm->nccl, st), "ncclRecv");
    }
    check_nccl(n.groupEnd(), "ncclGroupEnd");
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

void ll_comm_destroy(ll_comm* c) {
  if (!c) return;
  if (c->nccl) {
    try { ll::nccl().commDestroy(c->nccl); } catch (...) {}
  }
  delete c;
}

}  // extern "C"
