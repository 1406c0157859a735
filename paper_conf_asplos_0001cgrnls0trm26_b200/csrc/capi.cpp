// The C ABI of include/ll.h.  Every entry point converts internal errors into an
// ll_status and a thread-local message (nothing throws across the ABI).
#include <cuda_runtime.h>

#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <cctype>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <sstream>

#include "ll_internal.hpp"

namespace ll {
const std::string& last_error_ref();
std::string jit_precompile(const std::string& plan_src, const char* name);
int launch_generic(const void* src, void* dst, const unsigned long long* cols, int nbits, unsigned long long nelem,
                   int w, cudaStream_t stream, int sms);
void* copy_kernel_fn();
unsigned copy_kernel_grid(unsigned long long nbytes);
ll_status device_convert(const ConvPlan& P, const void* src, void* dst, void* ws, cudaStream_t st);
void plan_device(ConvPlan& P, const ll_plan_opts* opts);
}  // namespace ll

using namespace ll;

namespace {
// NVTX range around a host entry point (planning, launches): shows up in Nsight
// timelines; header-only NVTX v3, a no-op without a tool attached.
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

// Test / debugging hooks read at planning time:
//   LL_FORCE_CLASS=shuffle|smem  force the executed exchange when the caller's opts
//                                leave force_class automatic;
//   LL_LOG=1                     print every conversion plan (describe JSON) to stderr.
const ll_plan_opts* env_opts(const ll_plan_opts* opts, ll_plan_opts& tmp) {
  const char* e = std::getenv("LL_FORCE_CLASS");
  if (!e || !*e || (opts && opts->force_class >= 0)) return opts;
  if (opts) tmp = *opts; else ll_plan_opts_default(&tmp);
  std::string v(e);
  for (auto& c : v) c = char(std::tolower(static_cast<unsigned char>(c)));
  if (v == "shuffle") tmp.force_class = LL_CLASS_SHUFFLE;
  else if (v == "smem") tmp.force_class = LL_CLASS_SMEM;
  else return opts;
  return &tmp;
}
bool env_log() {
  const char* e = std::getenv("LL_LOG");
  return e && *e && std::string(e) != "0";
}
}  // namespace

#define LL_TRY try {
#define LL_CATCH                                                  \
  }                                                               \
  catch (const ll::Error& e) {                                    \
    set_last_error(e.what());                                     \
    return e.st;                                                  \
  }                                                               \
  catch (const std::bad_alloc&) {                                 \
    set_last_error("out of host memory");                         \
    return LL_ERR_OOM;                                            \
  }                                                               \
  catch (const std::exception& e) {                               \
    set_last_error(e.what());                                     \
    return LL_ERR_INVALID_ARG;                                    \
  }                                                               \
  return LL_OK;

namespace ll {

int num_sms() {
  static int sms = -1;
  if (sms < 0) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
      sms = 148;
  }
  return sms;
}

void check_cuda(cudaError_t e, const char* what) {
  if (e != cudaSuccess) fail(LL_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

// Launch of a specialised kernel with programmatic dependent launch (the kernels
// start with griddepcontrol.wait; ll_kernels.cuh ll_pdl_begin).  LL_PDL=0 disables.
void launch_kernel(void* kernel, unsigned grid, unsigned block, void** args, size_t smem, cudaStream_t st,
                   const char* what) {
  static const bool pdl = [] {
    const char* e = getenv("LL_PDL");
    return !(e && std::string(e) == "0");
  }();
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  check_cuda(cudaLaunchKernelExC(&cfg, kernel, args), what);
}

}  // namespace ll

namespace ll {
// 8-byte elements are converted as pairs of 4-byte atoms: a new lowest input bit
// maps to a new lowest logical bit (the product of the layout with a 1-bit identity,
// Def 4.3).  Packed buffers are unchanged byte-wise.
Layout atomize(const Layout& L) {
  Layout R;
  bool done = false;
  for (auto& d : L.in) {
    if (!done && (d.name == "reg" || d.name == "offset")) {
      R.in.push_back({d.name, d.bits + 1});
      done = true;
    } else {
      R.in.push_back(d);
    }
  }
  if (!done) R.in.insert(R.in.begin(), Dim{"reg", 1});
  R.out = L.out;
  R.out.push_back({"__atom", 1});
  // the new bit sits at position 0 of the first reg/offset dim, which is the first
  // dim in every supported layout; otherwise at the very front
  int pos = 0;
  {
    int p = 0;
    bool found = false;
    for (auto& d : L.in) {
      if (d.name == "reg" || d.name == "offset") { pos = p; found = true; break; }
      p += d.bits;
    }
    if (!found) pos = 0;
  }
  for (int k = 0; k < int(L.cols.size()); ++k) {
    if (k == pos) R.cols.push_back(1);
    R.cols.push_back(L.cols[k] << 1);
  }
  if (pos == int(L.cols.size())) R.cols.push_back(1);
  return R;
}

}  // namespace ll

namespace ll {
void ensure_tile_kernel(ConvPlan& P) {
  std::lock_guard<std::mutex> g(P.mu);
  if (P.kernel) return;
  if (P.source.empty()) P.source = codegen_tile(P);
  P.kernel = jit_kernel(P.source, P.peer_shift >= 0 ? "ll_tile_peer_kernel" : "ll_tile_kernel");
  if (P.smem_bytes > 48 * 1024)
    check_cuda(cudaFuncSetAttribute(P.kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, P.smem_bytes),
               "cudaFuncSetAttribute");
}

void ensure_gather_kernel(GatherPlan& G) {
  std::lock_guard<std::mutex> g(G.mu);
  if (G.kernel) return;
  G.kernel = jit_kernel(codegen_gather(G), "ll_gather_kernel");
  if (G.smem_bytes > 48 * 1024)
    check_cuda(cudaFuncSetAttribute(G.kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, G.smem_bytes),
               "cudaFuncSetAttribute");
}
}  // namespace ll

namespace {
int ilog2_u64(u64 v) { return v ? 63 - __builtin_clzll(v) : -1; }

unsigned grid_for(u64 ntiles) {
  const char* e = getenv("LL_GRID_PER_SM");
  int per = e ? atoi(e) : 0;
  u64 cap = per > 0 ? u64(num_sms()) * per : u64(0x7fffffff);
  u64 g = std::min<u64>(ntiles, cap);
  return unsigned(std::max<u64>(g, 1));
}

}  // namespace

namespace ll {
unsigned grid_for_tiles(u64 ntiles) { return grid_for(ntiles); }
}  // namespace ll

namespace ll {
ll_status convert_impl(const void* src, void* dst, void* ws, ConvPlan& P, cudaStream_t st) {
  const size_t sbytes = P.src_elems * P.w, dbytes = P.dst_elems * P.w;
  if ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15)
    fail(LL_ERR_MISALIGNED, "src and dst must be 16-byte aligned");
  const char* s8 = static_cast<const char*>(src);
  const char* d8 = static_cast<const char*>(dst);
  if (P.exec == EXEC_NOOP) {
    if (src == dst) return LL_OK;   // in place: nothing moves
    if (s8 < d8 + dbytes && d8 < s8 + sbytes) fail(LL_ERR_ALIAS, "NOOP: src and dst must be equal or disjoint");
    unsigned long long nb = dbytes;
    void* args[] = {const_cast<void**>(&src), &dst, &nb};
    launch_kernel(copy_kernel_fn(), copy_kernel_grid(nb), 256, args, 0, st, "cudaLaunchKernelEx(ll_copy_kernel)");
    return LL_OK;
  }
  if (s8 < d8 + dbytes && d8 < s8 + sbytes) fail(LL_ERR_ALIAS, "src and dst overlap (only NOOP plans may alias)");
  if (P.exec == EXEC_TILE) {
    ensure_tile_kernel(P);
    // data tiles x replica groups (broadcast replica bits above the unrolled ones)
    const size_t rep_grid = P.tile.rep_bits.size() - std::min<size_t>(size_t(P.tile.rep_lo), P.tile.rep_bits.size());
    u64 ntiles = u64(1) << (P.tile.grid_dst_bit.size() + rep_grid);
    unsigned long long nt = ntiles;
    void* args[] = {const_cast<void**>(&src), &dst, &nt};
    // staged tiles loop over their tiles with two stages in flight: a persistent grid
    const unsigned grid = (P.tile.staged || P.tile.bulk) ? unsigned(std::min<u64>(ntiles, u64(num_sms()))) : grid_for(ntiles);
    launch_kernel(P.kernel, grid, P.tile.threads(), args, size_t(P.smem_bytes), st,
                  "cudaLaunchKernelEx(ll_tile_kernel)");
    return LL_OK;
  }
  if (P.exec == EXEC_GENERIC) {
    const int nb = P.B.d_in() - (P.B.in_bits("dev"));
    std::vector<unsigned long long> cols(P.Q.begin(), P.Q.begin() + nb);
    int e = launch_generic(src, dst, cols.data(), nb, P.dst_elems, P.w, st, num_sms());
    check_cuda(cudaError_t(e), "ll_generic_convert_kernel");
    return LL_OK;
  }
  return device_convert(P, src, dst, ws, st);
}

}  // namespace ll

extern "C" {

const char* ll_last_error(void) { return ll::last_error_ref().c_str(); }
const char* ll_version(void) { return "ll-b200 0.1 (sm_100a)"; }

void ll_plan_opts_default(ll_plan_opts* o) {
  if (!o) return;
  std::memset(o, 0, sizeof *o);
  o->force_class = -1;
  o->max_vec_bytes = 16;
}

ll_status ll_layout_create(const ll_dim* in, int n_in, const ll_dim* out, int n_out, const int64_t* bases,
                           ll_layout** Lout) {
  LL_TRY
  if (!Lout || (n_in && !in) || (n_out && !out) || n_in < 0 || n_out < 0) fail(LL_ERR_INVALID_ARG, "null argument");
  auto* h = new ll_layout();
  std::unique_ptr<ll_layout> guard(h);
  Layout& L = h->L;
  int dout = 0;
  for (int i = 0; i < n_out; ++i) {
    if (!out[i].name || out[i].log2_size < 0 || out[i].log2_size > 62) fail(LL_ERR_INVALID_ARG, "bad output dim");
    L.out.push_back({out[i].name, out[i].log2_size});
    dout += out[i].log2_size;
  }
  int din = 0;
  for (int i = 0; i < n_in; ++i) {
    if (!in[i].name || in[i].log2_size < 0 || in[i].log2_size > 62) fail(LL_ERR_INVALID_ARG, "bad input dim");
    for (int j = 0; j < i; ++j)
      if (!std::strcmp(in[i].name, in[j].name)) fail(LL_ERR_INVALID_ARG, "duplicate input dim name");
    L.in.push_back({in[i].name, in[i].log2_size});
    din += in[i].log2_size;
  }
  if (din > 62 || dout > 62) fail(LL_ERR_INVALID_ARG, "more than 62 bits");
  if (din && !bases) fail(LL_ERR_INVALID_ARG, "null bases");
  for (int k = 0; k < din; ++k) {
    u64 f = 0;
    for (int i = 0; i < n_out; ++i) {
      int64_t c = bases[size_t(k) * n_out + i];
      if (c < 0 || (u64(c) >> L.out[i].bits)) fail(LL_ERR_INVALID_ARG, "basis coordinate out of range");
      f = (f << L.out[i].bits) | u64(c);
    }
    L.cols.push_back(f);
  }
  *Lout = guard.release();
  LL_CATCH
}

void ll_layout_destroy(ll_layout* L) { delete L; }

ll_status ll_layout_info(const ll_layout* L, int* n_in, int* n_out, int* d_in, int* d_out) {
  LL_TRY
  if (!L) fail(LL_ERR_INVALID_ARG, "null layout");
  if (n_in) *n_in = int(L->L.in.size());
  if (n_out) *n_out = int(L->L.out.size());
  if (d_in) *d_in = L->L.d_in();
  if (d_out) *d_out = L->L.d_out();
  LL_CATCH
}

ll_status ll_layout_dim(const ll_layout* L, int is_out, int index, const char** name, int* log2_size) {
  LL_TRY
  if (!L) fail(LL_ERR_INVALID_ARG, "null layout");
  auto& v = is_out ? L->L.out : L->L.in;
  if (index < 0 || index >= int(v.size())) fail(LL_ERR_INVALID_ARG, "dim index out of range");
  if (name) *name = v[index].name.c_str();
  if (log2_size) *log2_size = v[index].bits;
  LL_CATCH
}

ll_status ll_layout_bases(const ll_layout* L, int64_t* bases) {
  LL_TRY
  if (!L || !bases) fail(LL_ERR_INVALID_ARG, "null argument");
  const Layout& l = L->L;
  for (size_t k = 0; k < l.cols.size(); ++k)
    for (size_t i = 0; i < l.out.size(); ++i) {
      int sh = l.out_shift(int(i));
      bases[k * l.out.size() + i] = int64_t((l.cols[k] >> sh) & ((u64(1) << l.out[i].bits) - 1));
    }
  LL_CATCH
}

ll_status ll_layout_apply(const ll_layout* L, const int64_t* in_coords, int64_t* out_coords) {
  LL_TRY
  if (!L || !in_coords || !out_coords) fail(LL_ERR_INVALID_ARG, "null argument");
  const Layout& l = L->L;
  u64 h = 0;
  int s = 0;
  for (size_t i = 0; i < l.in.size(); ++i) {
    if (in_coords[i] < 0 || (u64(in_coords[i]) >> l.in[i].bits)) fail(LL_ERR_INVALID_ARG, "coordinate out of range");
    h |= u64(in_coords[i]) << s;
    s += l.in[i].bits;
  }
  u64 x = l.apply(h);
  for (size_t i = 0; i < l.out.size(); ++i)
    out_coords[i] = int64_t((x >> l.out_shift(int(i))) & ((u64(1) << l.out[i].bits) - 1));
  LL_CATCH
}

ll_status ll_layout_props(const ll_layout* L, int* surj, int* inj, int* dist, int* mem) {
  LL_TRY
  if (!L) fail(LL_ERR_INVALID_ARG, "null layout");
  if (surj) *surj = L->L.surjective();
  if (inj) *inj = L->L.injective();
  if (dist) *dist = L->L.distributed();
  if (mem) *mem = L->L.memory();
  LL_CATCH
}

ll_status ll_compose(const ll_layout* outer, const ll_layout* inner, ll_layout** out) {
  LL_TRY
  if (!outer || !inner || !out) fail(LL_ERR_INVALID_ARG, "null argument");
  auto* h = new ll_layout{compose(outer->L, inner->L)};
  *out = h;
  LL_CATCH
}

ll_status ll_invert(const ll_layout* L, ll_layout** out) {
  LL_TRY
  if (!L || !out) fail(LL_ERR_INVALID_ARG, "null argument");
  *out = new ll_layout{invert(L->L)};
  LL_CATCH
}

ll_status ll_product(const ll_layout* L1, const ll_layout* L2, ll_layout** out) {
  LL_TRY
  if (!L1 || !L2 || !out) fail(LL_ERR_INVALID_ARG, "null argument");
  *out = new ll_layout{product(L1->L, L2->L)};
  LL_CATCH
}

ll_status ll_left_divide(const ll_layout* M, const ll_layout* M1, ll_layout** M2) {
  LL_TRY
  if (!M || !M1 || !M2) fail(LL_ERR_INVALID_ARG, "null argument");
  *M2 = new ll_layout{left_divide(M->L, M1->L)};
  LL_CATCH
}

ll_status ll_kernel_basis(const ll_layout* L, int64_t* v, int* n) {
  LL_TRY
  if (!L || !v || !n) fail(LL_ERR_INVALID_ARG, "null argument");
  auto k = kernel_basis(L->L);
  for (size_t i = 0; i < k.size(); ++i) v[i] = int64_t(k[i]);
  *n = int(k.size());
  LL_CATCH
}

ll_status ll_layout_blocked(int rank, const int* shape, const int* size_per_thread, const int* threads_per_warp,
                            const int* warps_per_cta, const int* order, ll_layout** out) {
  LL_TRY
  if (rank < 1 || !shape || !size_per_thread || !threads_per_warp || !warps_per_cta || !order || !out)
    fail(LL_ERR_INVALID_ARG, "null argument");
  std::vector<int> sh(shape, shape + rank), s(size_per_thread, size_per_thread + rank),
      t(threads_per_warp, threads_per_warp + rank), w(warps_per_cta, warps_per_cta + rank), o(order, order + rank);
  std::vector<int> seen(rank, 0);
  for (int d : o) { if (d < 0 || d >= rank || seen[d]++) fail(LL_ERR_INVALID_ARG, "order must be a permutation"); }
  *out = new ll_layout{make_blocked(sh, s, t, w, o)};
  LL_CATCH
}

ll_status ll_layout_mma_acc(int M, int N, int warps_m, int warps_n, ll_layout** out) {
  LL_TRY
  if (!out) fail(LL_ERR_INVALID_ARG, "null argument");
  *out = new ll_layout{make_mma_acc(M, N, warps_m, warps_n)};
  LL_CATCH
}

ll_status ll_layout_mma_swizzle(int log2_rows, int log2_cols, int vec, int per_phase, int max_phase, ll_layout** out) {
  LL_TRY
  if (!out || log2_rows < 0 || log2_cols < 0 || log2_rows + log2_cols > 62) fail(LL_ERR_INVALID_ARG, "bad argument");
  *out = new ll_layout{make_mma_swizzle(log2_rows, log2_cols, vec, per_phase, max_phase)};
  LL_CATCH
}

ll_status ll_layout_contiguity(const ll_layout* L, int elem_bytes, int max_vec_bytes, int* elems) {
  LL_TRY
  if (!L || !elems || elem_bytes <= 0) fail(LL_ERR_INVALID_ARG, "bad argument");
  // the largest u with L^{-1}_Reg(i) = i for all i < u, i.e. the number of
  // leading register bits that map, in order, to logical flat bits 0, 1, 2, ...;
  // capped by the widest vector instruction (v4.b32).
  const Layout& l = L->L;
  int p = l.in_pos("reg"), nb = l.in_bits("reg"), k = 0;
  while (p >= 0 && k < nb && l.cols[p + k] == (u64(1) << k)) ++k;
  int cap = max_vec_bytes > 0 ? max_vec_bytes : 16;
  int e = 1 << k;
  while (e > 1 && e * elem_bytes > cap) e >>= 1;
  *elems = e;
  LL_CATCH
}

ll_status ll_layout_mma_operand(int is_rhs, int rows, int cols, int bitwidth, int warps_m, int warps_n,
                                ll_layout** out) {
  LL_TRY
  if (!out) fail(LL_ERR_INVALID_ARG, "null argument");
  *out = new ll_layout{make_mma_operand(is_rhs, rows, cols, bitwidth, warps_m, warps_n)};
  LL_CATCH
}

ll_status ll_layout_tmem_32x32b(int M, int N, ll_layout** out) {
  LL_TRY
  if (!out) fail(LL_ERR_INVALID_ARG, "null argument");
  *out = new ll_layout{make_tmem_32x32b(M, N)};
  LL_CATCH
}

ll_status ll_layout_tmem(const char* shape, int M, int N, ll_layout** out) {
  LL_TRY
  if (!out || !shape) fail(LL_ERR_INVALID_ARG, "null argument");
  *out = new ll_layout{make_tmem(shape, M, N)};
  LL_CATCH
}

ll_status ll_layout_slice(const ll_layout* L, int dim, ll_layout** out) {
  LL_TRY
  if (!L || !out) fail(LL_ERR_INVALID_ARG, "null argument");
  *out = new ll_layout{make_slice(L->L, dim)};
  LL_CATCH
}

namespace {
// Plan options shared by every planner: the vector bound must be a power of two in
// [1, 16] bytes (0 = default 16) — wider vectors have no ld/st instruction.
void validate_opts(const ll_plan_opts* o) {
  if (!o) return;
  const int v = o->max_vec_bytes;
  if (v < 0 || v > 16 || (v & (v - 1)) != 0)
    ll::fail(LL_ERR_INVALID_ARG, "max_vec_bytes must be 0 (default 16) or a power of two in [1, 16]");
}
}  // namespace

ll_status ll_plan_convert(const ll_layout* A, const ll_layout* B, int w, const ll_plan_opts* opts_in, ll_plan** plan) {
  LL_TRY
  NvtxRange nvtx("ll_plan_convert");
  if (!A || !B || !plan) fail(LL_ERR_INVALID_ARG, "null argument");
  ll_plan_opts opts_env;
  const ll_plan_opts* opts = env_opts(opts_in, opts_env);
  validate_opts(opts);
  auto h = std::make_unique<ll_plan>();
  h->kind = 0;
  if (w == 8) {
    // class of the original pair; execution on 4-byte atoms
    auto P0 = plan_convert(A->L, B->L, 8, opts);
    ll_class cls = P0->cls;
    if (P0->exec == EXEC_TILE || P0->exec == EXEC_GENERIC) {
      auto P = plan_convert(atomize(A->L), atomize(B->L), 4, opts);
      P->cls = cls;
      h->conv = std::move(P);
    } else {
      h->conv = std::move(P0);
    }
  } else {
    h->conv = plan_convert(A->L, B->L, w, opts);
  }
  if (h->conv->exec == EXEC_DEVICE) {
    plan_device(*h->conv, opts);
    ConvPlan* st[2] = {h->conv->pack.get(), h->conv->unpack.get()};
    for (int i = 0; i < 2; ++i)
      if (st[i]) {
        h->stage[i] = std::make_unique<ll_plan>();
        h->stage[i]->kind = 0;
        h->stage[i]->borrowed = st[i];
        if (st[i]->exec == EXEC_TILE) st[i]->source = codegen_tile(*st[i]);
      }
  }
  if (h->conv->exec == EXEC_TILE) h->conv->source = codegen_tile(*h->conv);
  if (env_log()) std::fprintf(stderr, "[ll] plan %s\n", describe(*h->conv).c_str());
  *plan = h.release();
  LL_CATCH
}

ll_status ll_plan_class(const ll_plan* p, ll_class* cls) {
  LL_TRY
  if (!p || !cls || p->kind != 0) fail(LL_ERR_INVALID_ARG, "not a conversion plan");
  *cls = p->cp().cls;
  LL_CATCH
}

ll_status ll_plan_workspace_bytes(const ll_plan* p, size_t* bytes) {
  LL_TRY
  if (!p || !bytes) fail(LL_ERR_INVALID_ARG, "null argument");
  *bytes = p->kind == 0 ? p->cp().workspace_bytes : 0;
  LL_CATCH
}

ll_status ll_plan_buffer_bytes(const ll_plan* p, size_t* src_bytes, size_t* dst_bytes, size_t* idx_bytes) {
  LL_TRY
  if (!p) fail(LL_ERR_INVALID_ARG, "null argument");
  auto local_bits = [](const Layout& L) {
    int n = 0;
    for (auto& d : L.in) if (d.name != "dev") n += d.bits;
    return n;
  };
  size_t s = 0, d = 0, i = 0;
  if (p->kind == 0) {
    const ConvPlan& P = p->cp();
    s = (size_t(1) << local_bits(P.A)) * size_t(P.w);
    d = (size_t(1) << local_bits(P.B)) * size_t(P.w);
  } else if (p->kind == 1) {
    const GatherPlan& G = *p->gather;
    s = d = (size_t(1) << local_bits(G.L)) * size_t(G.w);
    i = (size_t(1) << local_bits(G.L)) * 4;
  } else if (p->kind == 2) {
    s = (size_t(1) << local_bits(p->reduce->L)) * 4;
    d = size_t(p->reduce->out_elems) * 4;
  } else {
    s = d = (size_t(1) << local_bits(p->scan->L)) * 4;
  }
  if (src_bytes) *src_bytes = s;
  if (dst_bytes) *dst_bytes = d;
  if (idx_bytes) *idx_bytes = i;
  LL_CATCH
}

ll_status ll_plan_describe(const ll_plan* p, char* json, size_t cap) {
  LL_TRY
  if (!p || !json || !cap) fail(LL_ERR_INVALID_ARG, "null argument");
  std::string s;
  if (p->kind == 0) s = describe(p->cp());
  else if (p->kind == 1) {
    const GatherPlan& G = *p->gather;
    std::ostringstream o;
    o << "{\"kind\":\"gather\",\"sigma\":\"" << (G.sigma ? "faithful" : "coalesced") << "\",\"R\":" << G.R
      << ",\"warp_bits\":" << G.Wb << ",\"K_bits\":" << G.K_bits
      << ",\"exchange\":\"" << (G.smem ? "smem" : "shuffle") << "\",\"tma\":" << (G.tma ? "true" : "false") << ",\"tma_store\":" << (G.tma_store ? "true" : "false") << ",\"shuffles_per_elem\":" << (G.smem ? 0 : (1 << G.cand_bits))
      << ",\"ctas\":" << (u64(1) << G.grid_bit.size()) << "}";
    s = o.str();
  } else if (p->kind == 3) {
    const ScanPlan& S = *p->scan;
    std::ostringstream o;
    static const char* sopn[] = {"sum", "max", "min"};
    o << "{\"kind\":\"scan\",\"op\":\"" << sopn[S.op] << "\",\"sigma\":\"" << (S.sigma ? "faithful" : "coalesced") << "\",\"R\":" << S.R
      << ",\"warp_bits\":" << S.Wb << ",\"K_bits\":" << S.K_bits << ",\"steps\":" << S.K_bits
      << ",\"axis_hw\":" << "[";
    for (size_t t = 0; t < S.axis_hw.size(); ++t) o << (t ? "," : "") << S.axis_hw[t];
    o << "],\"shuffles_per_elem\":" << double(S.shfl_per_thread) / double(1 << S.R)
      << ",\"tma\":" << (S.tma ? "true" : "false") << ",\"tma_store\":" << (S.tma_store ? "true" : "false")
      << ",\"stages\":" << S.stages << ",\"smem_exchange_bytes\":" << S.xs_bytes
      << ",\"ctas\":" << (u64(1) << S.grid_bit.size()) << "}";
    s = o.str();
  } else {
    const ReducePlan& Rp = *p->reduce;
    std::ostringstream o;
    static const char* opn[] = {"sum", "max", "min"};
    o << "{\"kind\":\"reduce\",\"op\":\"" << opn[Rp.op] << "\",\"R\":" << Rp.R << ",\"warp_bits\":" << Rp.Wb << ",\"tree_levels\":" << Rp.red_reg.size()
      << ",\"bfly_stages\":" << Rp.red_lane.size() << ",\"warp_stages\":" << Rp.red_warp.size()
      << ",\"dup_bits\":" << Rp.dup_bits.size() << ",\"out_elems\":" << Rp.out_elems
      << ",\"axis_hw\":[";
    for (size_t t = 0; t < Rp.axis_hw.size(); ++t) o << (t ? "," : "") << Rp.axis_hw[t];
    o << "],\"shuffles_per_thread\":" << Rp.shfl_per_thread
      << ",\"tma\":" << (Rp.tma ? "true" : "false") << ",\"stages\":" << Rp.stages << ",\"sigma\":\"" << (Rp.sigma ? "faithful" : "coalesced") << "\""
      << ",\"ctas\":" << (u64(1) << Rp.grid_bit.size()) << "}";
    s = o.str();
  }
  std::strncpy(json, s.c_str(), cap - 1);
  json[cap - 1] = 0;
  if (s.size() >= cap) fail(LL_ERR_INVALID_ARG, "describe: buffer too small");
  LL_CATCH
}

ll_status ll_plan_source(const ll_plan* p, char* buf, size_t cap, size_t* needed) {
  LL_TRY
  if (!p) fail(LL_ERR_INVALID_ARG, "null plan");
  std::string s;
  if (p->kind == 0 && p->cp().exec == EXEC_TILE) s = p->cp().source;
  if (p->kind == 0 && p->cp().fused) s = p->cp().fused->source;
  if (p->kind == 1) s = codegen_gather(*p->gather);
  if (p->kind == 2) s = codegen_reduce(*p->reduce);
  if (p->kind == 3) s = codegen_scan(*p->scan);
  if (needed) *needed = s.size() + 1;
  if (buf && cap) {
    std::strncpy(buf, s.c_str(), cap - 1);
    buf[cap - 1] = 0;
  }
  LL_CATCH
}

ll_status ll_plan_prepare(ll_plan* p) {
  LL_TRY
  if (!p) fail(LL_ERR_INVALID_ARG, "null plan");
  if (p->kind == 0 && p->cp().exec == EXEC_TILE) ensure_tile_kernel(p->cp());
  if (p->kind == 0 && p->cp().exec == EXEC_DEVICE) {
    if (p->cp().pack && p->cp().pack->exec == EXEC_TILE) ensure_tile_kernel(*p->cp().pack);
    if (p->cp().unpack && p->cp().unpack->exec == EXEC_TILE) ensure_tile_kernel(*p->cp().unpack);
    if (p->cp().fused) ensure_tile_kernel(*p->cp().fused);
  }
  if (p->kind == 1) {
    ensure_gather_kernel(*p->gather);
  }
  if (p->kind == 3) {
    std::lock_guard<std::mutex> g(p->scan->mu);
    if (!p->scan->kernel) {
      p->scan->kernel = jit_kernel(codegen_scan(*p->scan), "ll_scan_kernel");
      if (p->scan->smem_bytes > 48 * 1024)
        check_cuda(cudaFuncSetAttribute(p->scan->kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        p->scan->smem_bytes), "cudaFuncSetAttribute");
    }
  }
  if (p->kind == 2) {
    std::lock_guard<std::mutex> g(p->reduce->mu);
    if (!p->reduce->kernel) {
      p->reduce->kernel = jit_kernel(codegen_reduce(*p->reduce), "ll_reduce_kernel");
      if (p->reduce->smem_bytes > 48 * 1024)
        check_cuda(cudaFuncSetAttribute(p->reduce->kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        p->reduce->smem_bytes), "cudaFuncSetAttribute");
    }
  }
  LL_CATCH
}

ll_status ll_jit_precompile(const ll_plan* p) {
  LL_TRY
  if (!p) fail(LL_ERR_INVALID_ARG, "null plan");
  if (p->kind == 0 && p->cp().exec == EXEC_TILE) jit_precompile(p->cp().source, "ll_tile_kernel");
  if (p->kind == 0 && p->cp().exec == EXEC_DEVICE) {
    const ConvPlan& P = p->cp();
    for (const ConvPlan* q : {P.pack.get(), P.unpack.get()})
      if (q && q->exec == EXEC_TILE) jit_precompile(q->source, "ll_tile_kernel");
    if (P.fused) jit_precompile(P.fused->source, "ll_tile_peer_kernel");
  }
  if (p->kind == 1) jit_precompile(codegen_gather(*p->gather), "ll_gather_kernel");
  if (p->kind == 2) jit_precompile(codegen_reduce(*p->reduce), "ll_reduce_kernel");
  if (p->kind == 3) jit_precompile(codegen_scan(*p->scan), "ll_scan_kernel");
  LL_CATCH
}

void ll_plan_destroy(ll_plan* p) {
  if (p && !p->borrowed) delete p;   // stage views are owned by their DEVICE plan
}

ll_status ll_convert(const void* src, void* dst, void* ws, const ll_plan* p, void* stream) {
  LL_TRY
  NvtxRange nvtx("ll_convert");
  if (!p || p->kind != 0) fail(LL_ERR_INVALID_ARG, "not a conversion plan");
  if (!src || !dst) fail(LL_ERR_INVALID_ARG, "null buffer");
  return convert_impl(src, dst, ws, p->cp(), static_cast<cudaStream_t>(stream));
  LL_CATCH
}

// Measured plan selection: every candidate kernel decomposition (thread_bytes 64 / 128
// / 256 and the default, with and without a forced smem exchange, with and without
// stmatrix / ldmatrix; for linear tiles also with and without the pipelined exchange
// and the two-CTAs-per-SM register cap) is planned,
// compiled and timed on the caller's buffers; the fastest plan is returned.
ll_status ll_plan_autotune(const ll_layout* A, const ll_layout* B, int w, const ll_plan_opts* base,
                           const void* src, void* dst, void* stream, int iters, ll_plan** out) {
  LL_TRY
  if (!A || !B || !out || !src || !dst) fail(LL_ERR_INVALID_ARG, "null argument");
  if (iters < 1) iters = 10;
  ll_plan_opts o0;
  if (base) o0 = *base; else ll_plan_opts_default(&o0);
  std::vector<ll_plan_opts> cand{o0};
  for (int tb : {64, 128, 256})
    if (o0.thread_bytes == 0) { ll_plan_opts c = o0; c.thread_bytes = tb; cand.push_back(c); }
  if (o0.force_class < 0) {
    const size_t nc = cand.size();
    for (size_t i = 0; i < nc; ++i) { ll_plan_opts c = cand[i]; c.force_class = LL_CLASS_SMEM; cand.push_back(c); }
  }
  // the layouts' own registers (faithful σ) against the coalesced decomposition: the
  // permuted fp8 operand shuffle measured 6656 vs 6365 GB/s faithful vs coalesced
  // (profiles/r02_sweep_eperm.jsonl); identical plans are timed once
  if (o0.sigma == SIGMA_COALESCED) { ll_plan_opts c = o0; c.sigma = SIGMA_FAITHFUL; cand.push_back(c); }
  // smem instructions (Thm 5.1): the automatic stmatrix / ldmatrix choice against
  // vectorised ld/st.shared only (identical plans are timed once)
  if (o0.smem_instr == 0) {
    const size_t nc = cand.size();
    for (size_t i = 0; i < nc; ++i) { ll_plan_opts c = cand[i]; c.smem_instr = 1; cand.push_back(c); }
  }
  // linear tiles (general invertible pull maps): the pipelined exchange and the ptxas
  // register cap (two CTAs per SM) both help some maps and hurt others — time them
  {
    ll_plan* raw = nullptr;
    if (ll_plan_convert(A, B, w, &o0, &raw) == LL_OK) {
      std::unique_ptr<ll_plan> p0(raw);
      const ConvPlan& P0 = p0->cp();
      if (P0.exec == EXEC_TILE && P0.tile.ld_run >= 0 && o0.pipe == 0 && o0.min_blocks == 0)
      {
        for (int pp : {1, 2})
          for (int mb : {-1, 2}) { ll_plan_opts c = o0; c.pipe = pp; c.min_blocks = mb; cand.push_back(c); }
        { ll_plan_opts c = o0; c.pipe = 3; c.min_blocks = -1; cand.push_back(c); }   // cp.async stages
        if (o0.tile_bytes == 0)   // 32 KiB tiles: shorter runs, lighter CTAs
          for (int mb : {0, -1}) { ll_plan_opts c = o0; c.tile_bytes = 32768; c.min_blocks = mb; cand.push_back(c); }
      }
    }
  }
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaEvent_t e0, e1;
  check_cuda(cudaEventCreate(&e0), "cudaEventCreate");
  check_cuda(cudaEventCreate(&e1), "cudaEventCreate");
  std::unique_ptr<ll_plan> best;
  float best_ms = 0;
  std::vector<std::string> seen;
  std::ostringstream log;
  log << "[";
  bool first = true;
  try {
    for (const ll_plan_opts& c : cand) {
      ll_plan* raw = nullptr;
      if (ll_plan_convert(A, B, w, &c, &raw) != LL_OK) continue;
      std::unique_ptr<ll_plan> p(raw);
      ConvPlan& P = p->cp();
      if (P.exec != EXEC_TILE) {          // nothing to tune: NOOP / generic / DEVICE
        if (!best) best = std::move(p);
        break;
      }
      if (std::find(seen.begin(), seen.end(), P.source) != seen.end()) continue;
      seen.push_back(P.source);
      convert_impl(src, dst, nullptr, P, st);   // compile, load, warm up
      convert_impl(src, dst, nullptr, P, st);
      check_cuda(cudaEventRecord(e0, st), "cudaEventRecord");
      for (int i = 0; i < iters; ++i) convert_impl(src, dst, nullptr, P, st);
      check_cuda(cudaEventRecord(e1, st), "cudaEventRecord");
      check_cuda(cudaEventSynchronize(e1), "cudaEventSynchronize");
      float ms = 0;
      check_cuda(cudaEventElapsedTime(&ms, e0, e1), "cudaEventElapsedTime");
      ms /= float(iters);
      static const char* xc[] = {"copy", "regperm", "shuffle", "smem"};
      log << (first ? "" : ",") << "{\"thread_bytes\":" << c.thread_bytes << ",\"tile_bytes\":" << c.tile_bytes
          << ",\"force_smem\":"
          << (c.force_class == LL_CLASS_SMEM ? "true" : "false") << ",\"smem_instr\":" << c.smem_instr
          << ",\"pipe\":" << (P.tile.pipe ? "true" : "false") << ",\"staged\":" << (P.tile.staged ? "true" : "false")
          << ",\"min_blocks\":" << P.tile.min_blocks
          << ",\"xchg\":\"" << xc[P.tile.xchg]
          << "\",\"R\":" << P.tile.R << ",\"threads\":" << P.tile.threads() << ",\"ms\":" << ms << "}";
      first = false;
      if (!best || ms < best_ms) { best = std::move(p); best_ms = ms; }
    }
  } catch (...) {
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    throw;
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (!best) fail(LL_ERR_UNSUPPORTED, "autotune: no candidate plan");
  log << "]";
  if (!first) best->cp().tune_json = log.str();
  *out = best.release();
  LL_CATCH
}

ll_status ll_convert_host(const void* src_host, void* dst_host, void* dev_buf, size_t dev_buf_bytes,
                          const ll_plan* p, int n_streams, void* const* streams) {
  LL_TRY
  if (!p || p->kind != 0 || !src_host || !dst_host || !dev_buf || n_streams < 1 || !streams)
    fail(LL_ERR_INVALID_ARG, "bad argument");
  ConvPlan& P = p->cp();
  if (P.exec != EXEC_TILE && P.exec != EXEC_NOOP)
    fail(LL_ERR_UNSUPPORTED, "ll_convert_host: tile or NOOP plans only (device / generic plans: use ll_convert)");
  const TilePlan& T = P.tile;
  // chunks are runs of whole CTA tiles, contiguous in both buffers: the grid bits must be
  // the top bits of src and dst, in the same order
  u64 ntiles = 1, tile_src = P.src_elems * P.w, tile_dst = P.dst_elems * P.w;
  if (P.exec == EXEC_TILE) {
    const size_t g = T.grid_dst_bit.size();
    int ns = int(ilog2_u64(P.src_elems)), nd = int(ilog2_u64(P.dst_elems));
    for (size_t k = 0; k < g; ++k)
      if (T.grid_src_bit[k] != ns - int(g) + int(k) || T.grid_dst_bit[k] != nd - int(g) + int(k))
        fail(LL_ERR_UNSUPPORTED, "ll_convert_host: the CTA grid is not the top bits of both buffers");
    // XOR (linear) grids: a chunk's tiles index their src by the global tile number, so
    // every grid column must be exactly its top src bit
    for (size_t k = 0; k < T.grid_src_xcol.size(); ++k)
      if (T.grid_src_xcol[k] != (u64(1) << T.grid_src_bit[k]))
        fail(LL_ERR_UNSUPPORTED, "ll_convert_host: the CTA grid's src columns are not plain top bits");
    ntiles = u64(1) << g;
    tile_src >>= g;
    tile_dst >>= g;
  }
  if (reinterpret_cast<uintptr_t>(dev_buf) & 15) fail(LL_ERR_MISALIGNED, "ll_convert_host: dev_buf must be 16-byte aligned");
  const u64 slot_bytes = (dev_buf_bytes / u64(n_streams)) & ~u64(255);   // 256-byte aligned slots
  u64 chunk = slot_bytes / (tile_src + tile_dst);
  if (chunk == 0) fail(LL_ERR_INVALID_ARG, "ll_convert_host: dev_buf too small for one tile per stream");
  chunk = std::min<u64>(chunk, std::max<u64>(1, ntiles / (2 * u64(n_streams))));   // >= 2 chunks per stream
  u64 c = 0;
  for (u64 t0 = 0; t0 < ntiles; t0 += chunk, ++c) {
    const u64 nt = std::min<u64>(chunk, ntiles - t0);
    cudaStream_t st = static_cast<cudaStream_t>(streams[c % u64(n_streams)]);
    char* slot = static_cast<char*>(dev_buf) + (c % u64(n_streams)) * slot_bytes;
    char* dsrc = slot;
    char* ddst = (P.exec == EXEC_NOOP) ? slot : slot + ((nt * tile_src + 15) & ~u64(15));
    check_cuda(cudaMemcpyAsync(dsrc, static_cast<const char*>(src_host) + t0 * tile_src, nt * tile_src,
                               cudaMemcpyHostToDevice, st), "cudaMemcpyAsync(H2D)");
    if (P.exec == EXEC_TILE) {
      ensure_tile_kernel(P);
      unsigned long long n = nt;
      void* args[] = {&dsrc, &ddst, &n};
      launch_kernel(P.kernel, grid_for(nt), T.threads(), args, size_t(P.smem_bytes), st,
                    "cudaLaunchKernelEx(ll_tile_kernel)");
    }
    check_cuda(cudaMemcpyAsync(static_cast<char*>(dst_host) + t0 * tile_dst, ddst, nt * tile_dst,
                               cudaMemcpyDeviceToHost, st), "cudaMemcpyAsync(D2H)");
  }
  LL_CATCH
}

ll_status ll_plan_gather(const ll_layout* L, int axis, int w, const ll_plan_opts* opts, ll_plan** plan) {
  LL_TRY
  if (!L || !plan) fail(LL_ERR_INVALID_ARG, "null argument");
  if (w == 8) fail(LL_ERR_UNSUPPORTED, "gather: elem_bytes 8 not supported");
  validate_opts(opts);
  auto h = std::make_unique<ll_plan>();
  h->kind = 1;
  h->gather = plan_gather(L->L, axis, w, opts);
  *plan = h.release();
  LL_CATCH
}

ll_status ll_gather(const void* src, const int32_t* idx, void* dst, const ll_plan* p, void* stream) {
  LL_TRY
  NvtxRange nvtx("ll_gather");
  if (!p || p->kind != 1) fail(LL_ERR_INVALID_ARG, "not a gather plan");
  if (!src || !idx || !dst) fail(LL_ERR_INVALID_ARG, "null buffer");
  if ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(idx) | reinterpret_cast<uintptr_t>(dst)) & 15)
    fail(LL_ERR_MISALIGNED, "buffers must be 16-byte aligned");
  GatherPlan& G = *p->gather;
  ensure_gather_kernel(G);
  unsigned long long nt = u64(1) << G.grid_bit.size();
  void* args[] = {const_cast<void**>(&src), const_cast<int32_t**>(&idx), &dst, &nt};
  // the TMA pipeline is persistent: as many CTAs as fit in shared memory per SM
  unsigned grid = grid_for(nt);
  if (G.tma) {
    u64 per_sm = std::max<u64>(1, std::min<u64>(8, (228u * 1024u) / u64(G.smem_bytes + 1024)));
    grid = unsigned(std::min<u64>(nt, per_sm * u64(num_sms())));
  }
  launch_kernel(G.kernel, grid, 32u << G.Wb, args, size_t(G.smem_bytes), static_cast<cudaStream_t>(stream),
                "cudaLaunchKernelEx(ll_gather_kernel)");
  LL_CATCH
}

ll_status ll_plan_scan(const ll_layout* L, int axis, const ll_plan_opts* opts, ll_plan** plan) {
  LL_TRY
  if (!L || !plan) fail(LL_ERR_INVALID_ARG, "null argument");
  validate_opts(opts);
  auto h = std::make_unique<ll_plan>();
  h->kind = 3;
  h->scan = plan_scan(L->L, axis, opts);
  *plan = h.release();
  LL_CATCH
}

ll_status ll_scan(const float* src, float* dst, const ll_plan* p, void* stream) {
  LL_TRY
  NvtxRange nvtx("ll_scan");
  if (!p || p->kind != 3) fail(LL_ERR_INVALID_ARG, "not a scan plan");
  if (!src || !dst) fail(LL_ERR_INVALID_ARG, "null buffer");
  if ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15)
    fail(LL_ERR_MISALIGNED, "buffers must be 16-byte aligned");
  ll_status st = ll_plan_prepare(const_cast<ll_plan*>(p));
  if (st != LL_OK) return st;
  ScanPlan& S = *p->scan;
  unsigned long long nt = u64(1) << S.grid_bit.size();
  void* args[] = {const_cast<float**>(&src), &dst, &nt};
  // the TMA pipeline is persistent: one CTA per SM streams its tiles through the stages
  unsigned grid = S.tma ? unsigned(std::min<u64>(nt, u64(num_sms()))) : grid_for(nt);
  launch_kernel(S.kernel, grid, 32u << S.Wb, args, size_t(S.smem_bytes), static_cast<cudaStream_t>(stream),
                "cudaLaunchKernelEx(ll_scan_kernel)");
  LL_CATCH
}

ll_status ll_plan_reduce(const ll_layout* L, int axis, const ll_plan_opts* opts, ll_plan** plan) {
  LL_TRY
  if (!L || !plan) fail(LL_ERR_INVALID_ARG, "null argument");
  validate_opts(opts);
  auto h = std::make_unique<ll_plan>();
  h->kind = 2;
  h->reduce = plan_reduce(L->L, axis, opts);
  *plan = h.release();
  LL_CATCH
}

ll_status ll_plan_reduce_out_elems(const ll_plan* p, size_t* n) {
  LL_TRY
  if (!p || p->kind != 2 || !n) fail(LL_ERR_INVALID_ARG, "not a reduce plan");
  *n = size_t(p->reduce->out_elems);
  LL_CATCH
}

ll_status ll_reduce(const float* src, float* dst, const ll_plan* p, void* stream) {
  LL_TRY
  NvtxRange nvtx("ll_reduce");
  if (!p || p->kind != 2) fail(LL_ERR_INVALID_ARG, "not a reduce plan");
  if (!src || !dst) fail(LL_ERR_INVALID_ARG, "null buffer");
  if (reinterpret_cast<uintptr_t>(src) & 15) fail(LL_ERR_MISALIGNED, "src must be 16-byte aligned");
  ll_status st = ll_plan_prepare(const_cast<ll_plan*>(p));
  if (st != LL_OK) return st;
  ReducePlan& Rp = *p->reduce;
  unsigned long long nt = u64(1) << Rp.grid_bit.size();
  void* args[] = {const_cast<float**>(&src), &dst, &nt};
  // the TMA pipeline is persistent: one CTA per SM streams its tiles through the stages
  unsigned grid = Rp.tma ? unsigned(std::min<u64>(nt, u64(num_sms()))) : grid_for(nt);
  launch_kernel(Rp.kernel, grid, 32u << Rp.Wb, args, size_t(Rp.smem_bytes), static_cast<cudaStream_t>(stream),
                "cudaLaunchKernelEx(ll_reduce_kernel)");
  LL_CATCH
}

ll_status ll_plan_device_stages(const ll_plan* p, ll_plan** pack, ll_plan** unpack, size_t* chunk_elems,
                                int* nranks) {
  LL_TRY
  if (!p || p->kind != 0) fail(LL_ERR_INVALID_ARG, "not a conversion plan");
  const ConvPlan& P = p->cp();
  if (P.exec != EXEC_DEVICE) fail(LL_ERR_INVALID_ARG, "not a DEVICE plan");
  if (pack) *pack = p->stage[0].get();
  if (unpack) *unpack = p->stage[1].get();
  if (chunk_elems) *chunk_elems = size_t(P.chunk_elems);
  if (nranks) *nranks = P.nranks;
  LL_CATCH
}

ll_status ll_plan_device_peers(const ll_plan* p, int rank, int* send_peers, int* recv_peers, int* nchunks) {
  LL_TRY
  if (!p || p->kind != 0 || !nchunks) fail(LL_ERR_INVALID_ARG, "bad argument");
  const ConvPlan& P = p->cp();
  if (P.exec != EXEC_DEVICE || P.exchange == LL_EXCHANGE_PEER) fail(LL_ERR_INVALID_ARG, "not a collective DEVICE plan");
  if (rank < 0 || rank >= P.nranks) fail(LL_ERR_INVALID_ARG, "rank out of range");
  const int n = 1 << P.xk;
  *nchunks = n;
  for (int j = 0; j < n; ++j) {
    if (send_peers) send_peers[j] = P.send_peer(u64(j), rank);
    if (recv_peers) recv_peers[j] = P.recv_peer(u64(j), rank);
  }
  LL_CATCH
}

ll_status ll_plan_simulate(const ll_plan* p, const void* src, void* dst) {
  LL_TRY
  if (!p || p->kind != 0 || !src || !dst) fail(LL_ERR_INVALID_ARG, "bad argument");
  // peer-exchange DEVICE plans: the fused tile plan over all ranks' slices back to back
  const ConvPlan& P = p->cp().fused ? *p->cp().fused : p->cp();
  if (P.exec != EXEC_TILE) fail(LL_ERR_UNSUPPORTED, "simulate: only tile plans");
  simulate_tile(P, static_cast<const uint8_t*>(src), static_cast<uint8_t*>(dst));
  LL_CATCH
}

}  // extern "C"
