// Linear layouts and their F2 algebra (row a2; Defs 4.1-4.5).
#include <algorithm>
#include <sstream>

#include "ll_internal.hpp"

namespace ll {

static thread_local std::string g_last_error;
void set_last_error(const std::string& m) { g_last_error = m; }
const std::string& last_error_ref() { return g_last_error; }
[[noreturn]] void fail(ll_status s, const std::string& msg) { throw Error(s, msg); }

int dim_level(const std::string& n) {
  if (n == "reg" || n == "register") return 0;
  if (n == "lane" || n == "thr" || n == "thread") return 1;
  if (n == "warp" || n == "wrp") return 2;
  if (n == "block" || n == "cta" || n == "offset") return 3;
  if (n == "dev" || n == "device") return 4;
  return -1;
}

int Layout::d_in() const { int s = 0; for (auto& d : in) s += d.bits; return s; }
int Layout::d_out() const { int s = 0; for (auto& d : out) s += d.bits; return s; }
int Layout::in_pos(const std::string& name) const {
  int p = 0;
  for (auto& d : in) { if (d.name == name) return p; p += d.bits; }
  return -1;
}
int Layout::in_bits(const std::string& name) const {
  for (auto& d : in) if (d.name == name) return d.bits;
  return 0;
}
int Layout::out_shift(int idx) const {
  int s = 0;
  for (size_t i = idx + 1; i < out.size(); ++i) s += out[i].bits;
  return s;
}
int Layout::rank() const {
  Echelon e;
  for (u64 c : cols) e.insert(c);
  return e.rank;
}
bool Layout::distributed() const {
  // Def 4.10: surjective; every column has at most one set bit; no
  // repeated non-zero columns.
  if (!surjective()) return false;
  std::vector<u64> nz;
  for (u64 c : cols) {
    if (popc(c) > 1) return false;
    if (c) nz.push_back(c);
  }
  std::sort(nz.begin(), nz.end());
  return std::adjacent_find(nz.begin(), nz.end()) == nz.end();
}
bool Layout::memory() const {
  // Def 4.14: invertible, columns with 1 or 2 set bits.
  if (d_in() != d_out() || !surjective()) return false;
  for (u64 c : cols) if (popc(c) < 1 || popc(c) > 2) return false;
  return true;
}
bool Layout::unit_columns() const {
  if (d_in() != d_out()) return false;
  u64 seen = 0;
  for (u64 c : cols) {
    if (popc(c) != 1 || (seen & c)) return false;
    seen |= c;
  }
  return true;
}

u64 apply_cols(const std::vector<u64>& cols, u64 v) {
  u64 x = 0;
  for (size_t k = 0; k < cols.size(); ++k) if ((v >> k) & 1) x ^= cols[k];
  return x;
}

std::vector<u64> right_inverse_cols(const Layout& L) {
  // Gaussian elimination over F2: process the columns in ascending order;
  // a column that reduces to zero is a free variable and stays 0 (slack = 0).
  Echelon e;
  for (size_t k = 0; k < L.cols.size(); ++k) e.insert(L.cols[k], u64(1) << k);
  if (e.rank != L.d_out()) fail(LL_ERR_NOT_SURJECTIVE, "layout is not surjective (P:194)");
  std::vector<u64> out(L.d_out());
  for (int t = 0; t < L.d_out(); ++t) {
    u64 c = 0;
    u64 r = e.reduce(u64(1) << t, &c);
    if (r) fail(LL_ERR_NOT_SURJECTIVE, "layout is not surjective (P:194)");
    out[t] = c;
  }
  return out;
}

std::vector<u64> kernel_basis(const Layout& L) {
  Echelon e;
  std::vector<u64> ker;
  for (size_t k = 0; k < L.cols.size(); ++k) {
    u64 c = u64(1) << k;
    u64 r = e.reduce(L.cols[k], &c);
    if (r) e.insert(r, c);      // (reduce again inside insert is a no-op)
    else ker.push_back(c);      // column k depends on earlier ones: kernel vector
  }
  return ker;
}

static u64 coords_to_flat(const std::vector<Dim>& dims, const std::vector<u64>& c) {
  u64 f = 0;
  for (size_t i = 0; i < dims.size(); ++i) f = (f << dims[i].bits) | c[i];
  return f;
}
static std::vector<u64> flat_to_coords(const std::vector<Dim>& dims, u64 f) {
  std::vector<u64> c(dims.size());
  for (int i = int(dims.size()) - 1; i >= 0; --i) {
    c[i] = dims[i].bits ? (f & ((u64(1) << dims[i].bits) - 1)) : 0;
    f = dims[i].bits >= 64 ? 0 : (f >> dims[i].bits);
  }
  return c;
}
static u64 hw_to_flat_hw(const std::vector<Dim>& dims, const std::vector<u64>& c) {
  // hardware flat: first dim least significant
  u64 h = 0; int s = 0;
  for (size_t i = 0; i < dims.size(); ++i) { h |= c[i] << s; s += dims[i].bits; }
  return h;
}
static std::vector<u64> hw_coords(const std::vector<Dim>& dims, u64 h) {
  std::vector<u64> c(dims.size());
  for (size_t i = 0; i < dims.size(); ++i) {
    c[i] = dims[i].bits ? (h & ((u64(1) << dims[i].bits) - 1)) : 0;
    h >>= dims[i].bits;
  }
  return c;
}

// Re-express a layout whose *output* is a hardware space (e.g. an inverse) — its
// output coordinates are the named dims, flattened row-major like any output.
Layout compose(const Layout& outer, const Layout& inner) {
  // Def 4.2: (outer ∘ inner)(u) = outer(inner(u)); label-wise matrix product.
  if (inner.out != outer.in) fail(LL_ERR_DIM_MISMATCH, "compose: inner.out != outer.in");
  Layout R;
  R.in = inner.in;
  R.out = outer.out;
  for (u64 c : inner.cols) {
    // c is a logical flat over inner.out (row-major); outer's input is hardware
    // flat (first dim lowest): convert coordinates.
    auto coords = flat_to_coords(inner.out, c);
    u64 h = hw_to_flat_hw(outer.in, coords);
    R.cols.push_back(outer.apply(h));
  }
  return R;
}

Layout invert(const Layout& L) {
  // Def 4.5: right inverse as a layout from L's output dims to L's input dims.
  auto hc = right_inverse_cols(L);   // per logical flat bit (lowest first)
  Layout R;
  R.in = L.out;
  R.out = L.in;
  // R's input bits in hardware-flat order: first dim of L.out lowest.  Logical
  // flat bit of (dim i, bit b) = out_shift(i) + b.
  for (size_t i = 0; i < L.out.size(); ++i) {
    int sh = L.out_shift(int(i));
    for (int b = 0; b < L.out[i].bits; ++b) {
      u64 h = hc[sh + b];
      R.cols.push_back(coords_to_flat(L.in, hw_coords(L.in, h)));
    }
  }
  return R;
}

static std::vector<Dim> merge_dims(const std::vector<Dim>& a, const std::vector<Dim>& b) {
  std::vector<Dim> r = a;
  for (auto& d : b) {
    bool found = false;
    for (auto& x : r) if (x.name == d.name) { x.bits += d.bits; found = true; }
    if (!found) r.push_back(d);
  }
  return r;
}

Layout product(const Layout& L1, const Layout& L2) {
  // Def 4.3, label-wise: dims with the same name concatenate, L1's
  // bits low; L2's images are shifted above L1's range in every output dim.
  Layout R;
  R.in = merge_dims(L1.in, L2.in);
  R.out = merge_dims(L1.out, L2.out);
  auto coord_in = [&](const Layout& S, u64 col, int shift_by_L1) {
    auto c = flat_to_coords(S.out, col);
    std::vector<u64> rc(R.out.size(), 0);
    for (size_t i = 0; i < S.out.size(); ++i) {
      size_t j = 0;
      while (R.out[j].name != S.out[i].name) ++j;
      int sh = 0;
      if (shift_by_L1)
        for (auto& d : L1.out) if (d.name == S.out[i].name) sh = d.bits;
      rc[j] = c[i] << sh;
    }
    return coords_to_flat(R.out, rc);
  };
  for (auto& d : R.in) {
    int p1 = L1.in_pos(d.name), b1 = L1.in_bits(d.name);
    int p2 = L2.in_pos(d.name), b2 = L2.in_bits(d.name);
    for (int k = 0; k < b1; ++k) R.cols.push_back(coord_in(L1, L1.cols[p1 + k], 0));
    for (int k = 0; k < b2; ++k) R.cols.push_back(coord_in(L2, L2.cols[p2 + k], 1));
  }
  return R;
}

Layout left_divide(const Layout& M, const Layout& M1) {
  // Def 4.4: M /_l M1 = M2 iff M = diag(M1, M2) label-wise.
  Layout R;
  for (auto& d : M.in) R.in.push_back({d.name, d.bits - M1.in_bits(d.name)});
  for (size_t i = 0; i < M.out.size(); ++i) {
    int b1 = 0;
    for (auto& d : M1.out) if (d.name == M.out[i].name) b1 = d.bits;
    R.out.push_back({M.out[i].name, M.out[i].bits - b1});
  }
  for (auto& d : R.in) if (d.bits < 0) fail(LL_ERR_NOT_DIVISIBLE, "M1 has more input bits than M");
  for (auto& d : R.out) if (d.bits < 0) fail(LL_ERR_NOT_DIVISIBLE, "M1 has more output bits than M");
  for (auto& d : M1.in) if (M.in_pos(d.name) < 0 && d.bits) fail(LL_ERR_NOT_DIVISIBLE, "M1 dim missing in M");
  for (auto& d : M.in) {
    int p = M.in_pos(d.name);
    int k1 = M1.in_bits(d.name);
    int p1 = M1.in_pos(d.name);
    for (int k = 0; k < d.bits; ++k) {
      auto c = flat_to_coords(M.out, M.cols[p + k]);
      if (k < k1) {
        auto c1 = flat_to_coords(M1.out, M1.cols[p1 + k]);
        for (size_t i = 0; i < M.out.size(); ++i) {
          u64 want = 0;
          for (size_t j = 0; j < M1.out.size(); ++j)
            if (M1.out[j].name == M.out[i].name) want = c1[j];
          if (c[i] != want) fail(LL_ERR_NOT_DIVISIBLE, "left division: low bits differ from M1");
        }
      } else {
        std::vector<u64> rc(M.out.size());
        for (size_t i = 0; i < M.out.size(); ++i) {
          int b1 = 0;
          for (auto& x : M1.out) if (x.name == M.out[i].name) b1 = x.bits;
          if (c[i] & ((u64(1) << b1) - 1)) fail(LL_ERR_NOT_DIVISIBLE, "left division: overlaps M1's range");
          rc[i] = c[i] >> b1;
        }
        R.cols.push_back(coords_to_flat(R.out, rc));
      }
    }
  }
  return R;
}

}  // namespace ll

// ---------------------------------------------------------------------------
// Layout families (§4.3; Props 9.1 / 9.2).  Output dims are "d0", "d1", ...
// (row-major, last fastest).
// ---------------------------------------------------------------------------
namespace ll {

static int lg2(int v) {
  if (v <= 0 || (v & (v - 1))) fail(LL_ERR_INVALID_ARG, "sizes must be powers of two (P:128)");
  return 31 - __builtin_clz(unsigned(v));
}

Layout make_blocked(const std::vector<int>& shape, const std::vector<int>& spt, const std::vector<int>& tpw,
                    const std::vector<int>& wpc, const std::vector<int>& order) {
  // Prop 9.1: σ_o^{-1} ∘ (id_R^o × id_T^o × id_W^o) — registers take sizePerThread in
  // `order` (fastest first), then lanes, then warps; if the CTA tile is smaller than the
  // shape the remaining bits become further registers in `order` (repetition); if it is
  // larger, the excess bits are zero columns (broadcast).
  const size_t nd = shape.size();
  if (spt.size() != nd || tpw.size() != nd || wpc.size() != nd || order.size() != nd)
    fail(LL_ERR_INVALID_ARG, "blocked: rank mismatch");
  Layout L;
  std::vector<int> sb(nd), used(nd, 0);
  for (size_t d = 0; d < nd; ++d) { sb[d] = lg2(shape[d]); L.out.push_back({"d" + std::to_string(d), sb[d]}); }
  auto flat_bit = [&](size_t d, int b) -> u64 {
    if (b >= sb[d]) return 0;
    int sh = 0;
    for (size_t e = d + 1; e < nd; ++e) sh += sb[e];
    return u64(1) << (sh + b);
  };
  auto take = [&](const std::vector<int>& cnt, std::vector<u64>& cols) {
    for (int d : order) for (int k = 0; k < lg2(cnt[d]); ++k) cols.push_back(flat_bit(d, used[d]++));
  };
  std::vector<u64> reg, lane, warp;
  take(spt, reg);
  take(tpw, lane);
  take(wpc, warp);
  for (int d : order) while (used[d] < sb[d]) reg.push_back(flat_bit(d, used[d]++));
  L.in = {{"reg", int(reg.size())}, {"lane", int(lane.size())}, {"warp", int(warp.size())}};
  L.cols = reg;
  L.cols.insert(L.cols.end(), lane.begin(), lane.end());
  L.cols.insert(L.cols.end(), warp.begin(), warp.end());
  return L;
}

Layout make_mma_acc(int M, int N, int warps_m, int warps_n) {
  // Prop 9.2 / G17: m16n8 accumulator fragment reg0->j0, lanes (j1,j2,i0,i1,i2),
  // reg1->i3; warps along M first (wgmma); n-repetitions then m-repetitions.
  const int mb = lg2(M), nb = lg2(N), wm = lg2(warps_m), wn = lg2(warps_n);
  auto I = [&](int k) -> u64 { return k < mb ? (u64(1) << (nb + k)) : 0; };
  auto J = [&](int k) -> u64 { return k < nb ? (u64(1) << k) : 0; };
  std::vector<u64> reg = {J(0), I(3)}, lane = {J(1), J(2), I(0), I(1), I(2)}, warp;
  for (int k = 0; k < wm; ++k) warp.push_back(I(4 + k));
  for (int k = 0; k < wn; ++k) warp.push_back(J(3 + k));
  for (int k = 3 + wn; k < nb; ++k) reg.push_back(J(k));
  for (int k = 4 + wm; k < mb; ++k) reg.push_back(I(k));
  Layout L;
  L.out = {{"d0", mb}, {"d1", nb}};
  L.in = {{"reg", int(reg.size())}, {"lane", 5}, {"warp", int(warp.size())}};
  L.cols = reg;
  L.cols.insert(L.cols.end(), lane.begin(), lane.end());
  L.cols.insert(L.cols.end(), warp.begin(), warp.end());
  return L;
}

Layout make_mma_swizzle(int m, int n, int vec, int per_phase, int max_phase) {
  // Def 4.11 as the memory layout offset -> (i, j): the matrix
  // [[I_n, C], [0, I_m]] with c_i = (vec · ((2^i / per_phase) mod max_phase)) mod 2^n;
  // the matrix is an involution, so it is both directions of the map.
  if (vec <= 0 || per_phase <= 0 || max_phase <= 0) fail(LL_ERR_INVALID_ARG, "swizzle parameters must be > 0");
  lg2(vec); lg2(per_phase); lg2(max_phase);
  Layout L;
  L.out = {{"d0", m}, {"d1", n}};
  L.in = {{"offset", m + n}};
  for (int k = 0; k < n; ++k) L.cols.push_back(u64(1) << k);
  for (int i = 0; i < m; ++i) {
    u64 c = (u64(vec) * u64(((u64(1) << i) / per_phase) % max_phase)) % (u64(1) << n);
    L.cols.push_back((u64(1) << (n + i)) | c);
  }
  return L;
}

Layout make_slice(const Layout& L, int dim) {
  // Prop 4.8: remove logical dim `dim` (Remark P:224: stays surjective, may gain zero
  // columns).
  if (dim < 0 || dim >= int(L.out.size())) fail(LL_ERR_INVALID_ARG, "slice: dim out of range");
  Layout R;
  R.in = L.in;
  for (int i = 0; i < int(L.out.size()); ++i) if (i != dim) R.out.push_back(L.out[i]);
  const int sh = L.out_shift(dim), b = L.out[dim].bits;
  const u64 lo = (u64(1) << sh) - 1;
  for (u64 c : L.cols) R.cols.push_back((c & lo) | ((c >> (sh + b)) << sh));
  return R;
}

}  // namespace ll

// ---------------------------------------------------------------------------
// MMA input operands (Prop 9.2) and the tcgen05 TMEM
// 32x32b load fragment (Blackwell tensor memory) as distributed layouts.
// ---------------------------------------------------------------------------
namespace ll {

Layout make_mma_operand(int is_rhs, int rows, int cols, int bitwidth, int warps_m, int warps_n) {
  // lhs (M x K, d0 = m, d1 = k):
  //   id^{Reg,1}_{log2(32/b)} x id^{Thr,1}_2 x id^{Thr,0}_3 x id^{Reg,0}_1 x id^{Reg,1}_1
  // rhs (K x N, d0 = k, d1 = n):
  //   id^{Reg,0}_{log2(32/b)} x id^{Thr,0}_2 x id^{Thr,1}_3 x id^{Reg,1}_1
  // then repetitions over the k dim, then the other dim, as register bits; warps along
  // M then N: the operand's own dim is split, warps on the other dim broadcast (zero
  // columns).
  if (bitwidth != 8 && bitwidth != 16 && bitwidth != 32) fail(LL_ERR_INVALID_ARG, "operand bitwidth must be 8, 16 or 32");
  const int rb = lg2(rows), cb = lg2(cols), kb = lg2(32 / bitwidth);
  const int wm = lg2(warps_m), wn = lg2(warps_n);
  // dims: lhs (d0 = m, d1 = k); rhs (d0 = k, d1 = n)
  auto D0 = [&](int k) -> u64 { return k < rb ? (u64(1) << (cb + k)) : 0; };
  auto D1 = [&](int k) -> u64 { return k < cb ? (u64(1) << k) : 0; };
  std::vector<u64> reg, lane, warp;
  int k_used = 0, o_used = 0;   // bits used on the k dim / the other dim
  auto K = [&](int k) { return is_rhs ? D0(k) : D1(k); };
  auto Oth = [&](int k) { return is_rhs ? D1(k) : D0(k); };
  for (int t = 0; t < kb; ++t) reg.push_back(K(k_used++));
  for (int t = 0; t < 2; ++t) lane.push_back(K(k_used++));
  for (int t = 0; t < 3; ++t) lane.push_back(Oth(o_used++));
  if (!is_rhs) { reg.push_back(Oth(o_used++)); }   // rows +8 (lhs only: 16-row tile)
  reg.push_back(K(k_used++));                      // k + 8·(32/b)/... second k half
  // warps: lhs splits M (i) over warps_m, broadcasts over warps_n; rhs the converse
  for (int t = 0; t < wm; ++t) warp.push_back(is_rhs ? 0 : Oth(o_used++));
  for (int t = 0; t < wn; ++t) warp.push_back(is_rhs ? Oth(o_used++) : 0);
  const int kdim_bits = is_rhs ? rb : cb, odim_bits = is_rhs ? cb : rb;
  while (k_used < kdim_bits) reg.push_back(K(k_used++));
  while (o_used < odim_bits) reg.push_back(Oth(o_used++));
  Layout L;
  L.out = {{"d0", rb}, {"d1", cb}};
  L.in = {{"reg", int(reg.size())}, {"lane", 5}, {"warp", int(warp.size())}};
  L.cols = reg;
  L.cols.insert(L.cols.end(), lane.begin(), lane.end());
  L.cols.insert(L.cols.end(), warp.begin(), warp.end());
  return L;
}

Layout make_tmem_32x32b(int M, int N) {
  // tcgen05.ld.32x32b: warp w of a warpgroup reads TMEM lanes [32w, 32w + 32); thread
  // t gets lane (row) 32w + t; consecutive registers are consecutive columns.
  const int mb = lg2(M), nb = lg2(N);
  if (mb != 7) fail(LL_ERR_INVALID_ARG, "tmem 32x32b fragment: M must be 128 (4 warps x 32 lanes)");
  Layout L;
  L.out = {{"d0", mb}, {"d1", nb}};
  L.in = {{"reg", nb}, {"lane", 5}, {"warp", 2}};
  for (int k = 0; k < nb; ++k) L.cols.push_back(u64(1) << k);
  for (int k = 0; k < 7; ++k) L.cols.push_back(u64(1) << (nb + k));
  return L;
}

// tcgen05.ld fragment families: a warpgroup loads the 128 x N fp32
// accumulator (TMEM lane = row, 32-bit TMEM column = column); warp w owns lanes
// [32w, 32w + 32).  One x1 load per warp covers (lanes x columns):
//   32x32b  32 x 1   thread -> row (5 bits)
//   16x64b  16 x 2   thread bits (row 3, col 0, row 0, row 1, row 2)
//   16x128b 16 x 4   thread bits (col 0, col 1, row 0-2); register -> row 3
//   16x256b 16 x 8   thread bits (col 1, col 2, row 0-2); registers (col 0, row 3)
// then .x<num> repetitions along the columns (register bits), the second 16-lane load
// of the 16-row shapes (register bit -> row 4), and the warps (rows 5, 6).
Layout make_tmem(const std::string& shape, int M, int N) {
  const int mb = lg2(M), nb = lg2(N);
  if (mb != 7) fail(LL_ERR_INVALID_ARG, "tmem fragment: M must be 128 (a warpgroup's 128 TMEM lanes)");
  auto row = [&](int k) { return u64(1) << (nb + k); };
  auto col = [&](int k) { return k < nb ? u64(1) << k : u64(0); };
  std::vector<u64> reg, lane;
  int x1_cols;   // log2 of the columns one x1 load covers
  bool half = true;
  if (shape == "32x32b") {
    for (int k = 0; k < 5; ++k) lane.push_back(row(k));
    x1_cols = 0;
    half = false;
  } else if (shape == "16x64b") {
    lane = {row(3), col(0), row(0), row(1), row(2)};
    x1_cols = 1;
  } else if (shape == "16x128b") {
    reg = {row(3)};
    lane = {col(0), col(1), row(0), row(1), row(2)};
    x1_cols = 2;
  } else if (shape == "16x256b") {
    reg = {col(0), row(3)};
    lane = {col(1), col(2), row(0), row(1), row(2)};
    x1_cols = 3;
  } else {
    fail(LL_ERR_INVALID_ARG, "tmem fragment shape must be 32x32b, 16x64b, 16x128b or 16x256b");
  }
  if (nb < x1_cols) fail(LL_ERR_INVALID_ARG, "tmem fragment: N smaller than one x1 load");
  for (int k = x1_cols; k < nb; ++k) reg.push_back(col(k));
  if (half) reg.push_back(row(4));
  Layout L;
  L.out = {{"d0", mb}, {"d1", nb}};
  L.in = {{"reg", int(reg.size())}, {"lane", 5}, {"warp", 2}};
  L.cols = reg;
  L.cols.insert(L.cols.end(), lane.begin(), lane.end());
  L.cols.push_back(row(5));
  L.cols.push_back(row(6));
  return L;
}

}  // namespace ll
