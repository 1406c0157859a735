// Conversion planner (rows a3, a4, a6-a9) plus gather (a11) and
// reduce (a12) plans.
#include <algorithm>
#include <cstdlib>
#include <functional>
#include <cstring>
#include <sstream>

#include "ll_internal.hpp"

namespace ll {

namespace {

int ilog2(u64 v) { return v ? lead(v) : -1; }

int default_int(const ll_plan_opts* o, int ll_plan_opts::*f, int dflt) {
  if (!o) return dflt;
  int v = o->*f;
  return v > 0 ? v : dflt;
}

// Bits of the layout belonging to dims of level <= maxlev / == lev.
std::vector<int> bits_at_level(const Layout& L, int lev_lo, int lev_hi) {
  std::vector<int> r;
  int p = 0;
  for (auto& d : L.in) {
    int lv = dim_level(d.name);
    if (lv >= lev_lo && lv <= lev_hi)
      for (int k = 0; k < d.bits; ++k) r.push_back(p + k);
    p += d.bits;
  }
  return r;
}

int dev_bits(const Layout& L) { return L.in_bits("dev") + L.in_bits("device"); }

}  // namespace

// ---------------------------------------------------------------------------
// Pull map and class.  Q[k] = A^+(B.col[k]) with the slack-zero right
// inverse (rule (2)).  The class is the lowest level λ such that Q can be
// adjusted by ker(A) (a choice of preimage) to be the identity on every input dim
// above λ (rule (1)) — equal to the existential class of SURVEY O7.
// ---------------------------------------------------------------------------
static int classify_and_adjust(const Layout& A, const Layout& B, std::vector<u64>& Q) {
  auto Ainv = right_inverse_cols(A);
  Q.assign(B.cols.size(), 0);
  for (size_t k = 0; k < B.cols.size(); ++k) Q[k] = apply_cols(Ainv, B.cols[k]);
  auto ker = kernel_basis(A);
  for (int lev = 0; lev <= 4; ++lev) {
    // high-dim mask of A and, for each B bit in a high dim, its A counterpart
    u64 hiA = 0;
    int p = 0;
    for (auto& d : A.in) {
      if (dim_level(d.name) > lev) for (int t = 0; t < d.bits; ++t) hiA |= u64(1) << (p + t);
      p += d.bits;
    }
    bool ok = true;
    std::vector<u64> target(B.cols.size(), 0);
    p = 0;
    for (auto& d : B.in) {
      if (dim_level(d.name) > lev) {
        int pa = A.in_pos(d.name), ba = A.in_bits(d.name);
        for (int t = 0; t < d.bits; ++t) {
          if (pa < 0 || t >= ba) { ok = false; break; }
          target[p + t] = u64(1) << (pa + t);
        }
      }
      if (!ok) break;
      p += d.bits;
    }
    if (!ok) continue;
    Echelon ek;
    for (size_t i = 0; i < ker.size(); ++i) ek.insert(ker[i] & hiA, u64(1) << i);
    std::vector<u64> adj(Q.size());
    for (size_t k = 0; k < Q.size() && ok; ++k) {
      u64 delta = (Q[k] & hiA) ^ target[k];
      u64 c = 0;
      if (ek.reduce(delta, &c)) { ok = false; break; }
      u64 fix = 0;
      for (size_t i = 0; i < ker.size(); ++i) if ((c >> i) & 1) fix ^= ker[i];
      adj[k] = Q[k] ^ fix;
    }
    if (!ok) continue;
    Q = adj;
    return lev;
  }
  fail(LL_ERR_UNSUPPORTED, "no class found (internal)");
}

// ---------------------------------------------------------------------------
// Kernel decomposition (σ_ld, σ_st) of a permutation Q over one CTA tile.
//   S: src packed bits of the tile (ascending), D: dst packed bits (ascending);
//   colA(s) = A.cols[s], colB(d) = B.cols[d]; the two sets of logical vectors are
//   equal.  prefer_warp: logical vectors preferred as kernel warps (in order).
// Coalesced σ: kreg[0, v) = lowest v tile bits (one 16-byte
// vector), klane = the next 5 bits (a warp instruction covers 512 contiguous
// bytes), kernel warps = common vectors where possible, remaining bits -> regs.
// ---------------------------------------------------------------------------
static void assign_sigma_coalesced(TilePlan& T, const Layout& A, const Layout& B,
                                   const std::vector<int>& S, const std::vector<int>& D,
                                   const std::vector<u64>& prefer_warp, int maxvec, int thread_bytes) {
  const int n = int(S.size());
  const int w = T.w;
  T.n = n;
  int R = std::max(0, ilog2(std::max(1, thread_bytes / w)));
  int Wb = n - 5 - R;
  if (Wb < 0) Wb = 0;
  if (Wb > 5) Wb = 5;
  R = n - 5 - Wb;
  if (R < 0) fail(LL_ERR_UNSUPPORTED, "tile smaller than one warp");
  T.R = R;
  T.Wb = Wb;
  int v = std::min(std::max(0, ilog2(std::max(1, maxvec / w))), R);
  // a global vector needs its v bits to be the packed positions 0..v-1 (broadcast
  // layouts may skip a low position: then the vector shrinks to the contiguous prefix)
  int vl = 0, vs = 0;
  while (vl < v && S[vl] == vl) ++vl;
  while (vs < v && D[vs] == vs) ++vs;
  T.vld = vl;
  T.vst = vs;
  T.ld_bit.assign(n, -1);
  T.st_bit.assign(n, -1);
  for (int b = 0; b < v; ++b) { T.ld_bit[b] = S[b]; T.st_bit[b] = D[b]; }
  for (int t = 0; t < 5; ++t) { T.ld_bit[R + t] = S[v + t]; T.st_bit[R + t] = D[v + t]; }
  std::vector<int> restS(S.begin() + v + 5, S.end()), restD(D.begin() + v + 5, D.end());
  auto findS = [&](u64 c) { for (size_t i = 0; i < restS.size(); ++i) if (A.cols[restS[i]] == c) return int(i); return -1; };
  auto findD = [&](u64 c) { for (size_t i = 0; i < restD.size(); ++i) if (B.cols[restD[i]] == c) return int(i); return -1; };
  // 1. vectorisation set: logical vectors that can be register bits on
  //    both sides — the forced low registers of one side placed among the free
  //    registers of the other — in A's register order, within max_vec_bytes (G9).
  std::vector<int> regS, regD;   // free register bits reserved for Vec (packed bits)
  {
    std::vector<u64> order;
    for (int b = 0; b < v; ++b) order.push_back(A.cols[S[b]]);
    for (int b = 0; b < v; ++b) order.push_back(B.cols[D[b]]);
    auto forcedA = [&](u64 c) { for (int b = 0; b < v; ++b) if (A.cols[S[b]] == c) return true; return false; };
    auto forcedB = [&](u64 c) { for (int b = 0; b < v; ++b) if (B.cols[D[b]] == c) return true; return false; };
    int nv = 0;
    const int free_regs = R - v;
    std::vector<u64> chosen;
    for (u64 c : order) {
      if ((2 << nv) * w > maxvec) break;
      if (std::find(chosen.begin(), chosen.end(), c) != chosen.end()) continue;
      bool inA = forcedA(c), inB = forcedB(c);
      if (inA && inB) { ++nv; chosen.push_back(c); continue; }
      int is = inA ? -1 : findS(c), id = inB ? -1 : findD(c);
      if ((!inA && (is < 0 || int(regS.size()) >= free_regs)) || (!inB && (id < 0 || int(regD.size()) >= free_regs)))
        continue;
      if (!inA) { regS.push_back(restS[is]); restS.erase(restS.begin() + is); }
      if (!inB) { regD.push_back(restD[id]); restD.erase(restD.begin() + id); }
      ++nv;
      chosen.push_back(c);
    }
  }
  // 2. kernel warps: common logical vectors first (preferred ones, then ascending src
  //    position), so that warp-level classes (SHUFFLE/REGPERM) stay available
  std::vector<u64> cand = prefer_warp;
  for (int s : restS) cand.push_back(A.cols[s]);
  int wi = 0;
  for (u64 c : cand) {
    if (wi == Wb) break;
    int is = findS(c), id = findD(c);
    if (is < 0 || id < 0) continue;
    T.ld_bit[R + 5 + wi] = restS[is];
    T.st_bit[R + 5 + wi] = restD[id];
    restS.erase(restS.begin() + is);
    restD.erase(restD.begin() + id);
    ++wi;
  }
  // not enough common vectors: take the highest remaining bits on each side
  while (wi < Wb) {
    T.ld_bit[R + 5 + wi] = restS.back(); restS.pop_back();
    T.st_bit[R + 5 + wi] = restD.back(); restD.pop_back();
    ++wi;
  }
  // 3. remaining register bits: reserved Vec bits first, then ascending
  std::sort(restS.begin(), restS.end());
  std::sort(restD.begin(), restD.end());
  regS.insert(regS.end(), restS.begin(), restS.end());
  regD.insert(regD.end(), restD.begin(), restD.end());
  for (int b = v; b < R; ++b) { T.ld_bit[b] = regS[b - v]; T.st_bit[b] = regD[b - v]; }
  T.sigma = SIGMA_COALESCED;
}

static void assign_sigma_faithful(TilePlan& T, const Layout& A, const Layout& B,
                                  const std::vector<int>& foldS, const std::vector<int>& foldD, int maxvec) {
  // kernel hardware = A's (reg, lane, warp) for loads and B's for stores, plus
  // folded block bits as extra warps.
  auto reg = [](const Layout& L, const char* nm) {
    std::vector<int> r; int p = L.in_pos(nm);
    for (int k = 0; k < L.in_bits(nm); ++k) r.push_back(p + k);
    return r;
  };
  auto rA = reg(A, "reg"), lA = reg(A, "lane"), wA = reg(A, "warp");
  auto rB = reg(B, "reg"), lB = reg(B, "lane"), wB = reg(B, "warp");
  if (lA.size() != 5 || lB.size() != 5 || rA.size() != rB.size() || wA.size() != wB.size())
    fail(LL_ERR_UNSUPPORTED, "faithful σ needs 5 lane bits and equal reg/warp sizes");
  T.R = int(rA.size());
  T.Wb = int(wA.size() + foldS.size());
  T.n = T.R + 5 + T.Wb;
  if (T.Wb > 5) fail(LL_ERR_UNSUPPORTED, "too many warps");
  T.ld_bit.clear(); T.st_bit.clear();
  for (int b : rA) T.ld_bit.push_back(b);
  for (int b : lA) T.ld_bit.push_back(b);
  for (int b : wA) T.ld_bit.push_back(b);
  for (int b : foldS) T.ld_bit.push_back(b);
  for (int b : rB) T.st_bit.push_back(b);
  for (int b : lB) T.st_bit.push_back(b);
  for (int b : wB) T.st_bit.push_back(b);
  for (int b : foldD) T.st_bit.push_back(b);
  int v = std::min(std::max(0, ilog2(std::max(1, maxvec / T.w))), T.R);
  T.vld = T.vst = v;
  T.sigma = SIGMA_FAITHFUL;
}

// ---------------------------------------------------------------- exchange plans
static void plan_regperm(TilePlan& T) {
  // (B^{-1}∘A)_Reg is a register permutation: out slot e holds the
  // logical element of L_st slot e, found in the L_ld slot with the same register
  // logical vectors (lanes and warps agree).
  std::vector<int> map(T.R, -1);
  for (int b = 0; b < T.R; ++b)
    for (int a = 0; a < T.R; ++a)
      if (T.lcol_ld[a] == T.lcol_st[b]) map[b] = a;
  for (int b = 0; b < T.R; ++b)
    if (map[b] < 0) fail(LL_ERR_UNSUPPORTED, "regperm: register sets differ (internal)");
  T.perm.assign(size_t(1) << T.R, 0);
  for (u64 e = 0; e < (u64(1) << T.R); ++e) {
    u64 s = 0;
    for (int b = 0; b < T.R; ++b) if ((e >> b) & 1) s |= u64(1) << map[b];
    T.perm[e] = int(s);
  }
}

// Fit f(l) = c ⊕ Σ_t l_t·col_t over lane bits; returns false if f is not affine.
static bool fit_affine(const std::vector<int>& f, int& c, int col[5]) {
  c = f[0];
  for (int t = 0; t < 5; ++t) col[t] = f[1 << t] ^ c;
  for (int l = 0; l < 32; ++l) {
    int g = c;
    for (int t = 0; t < 5; ++t) if ((l >> t) & 1) g ^= col[t];
    if (g != f[l]) return false;
  }
  return true;
}

// Conditional-swap stages realising "slot j <- slot j ⊕ (Σ_t l_t col_t)".
// The stages use a basis of span{col_t}; lane bit t's mask is expressed in it, and
// stage i fires on the parity of the lane bits whose expression contains basis vector i.
static void xor_network(const int col[5], std::vector<uint32_t>& lmask, std::vector<int>& xs) {
  Echelon e2;
  std::vector<u64> orig;
  for (int t = 0; t < 5; ++t)
    if (col[t] && e2.insert(u64(col[t]), u64(1) << orig.size())) orig.push_back(u64(col[t]));
  lmask.assign(orig.size(), 0);
  xs.assign(orig.size(), 0);
  for (size_t i = 0; i < orig.size(); ++i) xs[i] = int(orig[i]);
  for (int t = 0; t < 5; ++t) {
    if (!col[t]) continue;
    u64 c = 0;
    e2.reduce(u64(col[t]), &c);   // col[t] = Σ_i c_i orig[i]
    for (size_t i = 0; i < orig.size(); ++i) if ((c >> i) & 1) lmask[i] |= 1u << t;
  }
}

static bool plan_shuffle(TilePlan& T) {
  // P:371-389 on the kernel layouts L_ld -> L_st within one warp.
  const int R = T.R, w = T.w;
  const int u = w < 4 ? ilog2(4 / w) : 0;        // reg bits inside one 32-bit unit
  if (u > R) return false;
  for (int b = 0; b < u; ++b) if (T.lcol_ld[b] != T.lcol_st[b]) return false;   // word units
  T.unit_elems = 1 << u;
  T.nslot = 1 << (R - u);
  // V: the common register vectors forming one 32-bit unit.
  T.V.assign(T.lcol_ld.begin(), T.lcol_ld.begin() + u);
  std::vector<u64> aThr(T.lcol_ld.begin() + R, T.lcol_ld.begin() + R + 5);
  std::vector<u64> bThr(T.lcol_st.begin() + R, T.lcol_st.begin() + R + 5);
  T.I.clear(); T.E.clear(); T.F.clear(); T.G.clear(); T.Rb.clear();
  for (u64 c : aThr) if (std::find(bThr.begin(), bThr.end(), c) != bThr.end()) T.I.push_back(c);
  for (u64 c : aThr) if (std::find(T.I.begin(), T.I.end(), c) == T.I.end()) T.E.push_back(c);
  for (u64 c : bThr) if (std::find(T.I.begin(), T.I.end(), c) == T.I.end()) T.F.push_back(c);
  std::sort(T.E.begin(), T.E.end());     // "ascending order" (G8)
  std::sort(T.F.begin(), T.F.end());
  if (T.E.size() != T.F.size()) return false;
  for (size_t i = 0; i < T.E.size(); ++i) T.G.push_back(T.E[i] ^ T.F[i]);
  // R completes V ∪ I ∪ G to the warp space
  Echelon ech;
  for (u64 c : T.V) ech.insert(c);
  for (u64 c : T.I) ech.insert(c);
  for (u64 c : T.G) ech.insert(c);
  std::vector<u64> wsp(T.lcol_ld.begin(), T.lcol_ld.begin() + R + 5);
  std::sort(wsp.begin(), wsp.end());
  for (u64 c : wsp) if (ech.insert(c)) T.Rb.push_back(c);
  T.rounds = 1 << T.Rb.size();
  if (T.rounds != T.nslot) return false;
  // inverse maps logical -> (reg, lane) for L_ld and L_st (within the warp)
  auto inv_of = [&](const std::vector<u64>& lc) {
    Echelon e;
    for (int b = 0; b < R + 5; ++b) e.insert(lc[b], u64(1) << b);
    return e;
  };
  Echelon invLd = inv_of(T.lcol_ld), invSt = inv_of(T.lcol_st);
  auto hw_of = [&](const Echelon& e, u64 x) {
    u64 c = 0;
    if (e.reduce(x, &c)) fail(LL_ERR_UNSUPPORTED, "shuffle: element outside warp space");
    return c;
  };
  // span(V ∪ I ∪ G) enumerated once
  std::vector<u64> gens = T.V;
  gens.insert(gens.end(), T.I.begin(), T.I.end());
  gens.insert(gens.end(), T.G.begin(), T.G.end());
  std::vector<u64> spanv(size_t(1) << gens.size(), 0);
  for (size_t m = 1; m < spanv.size(); ++m) {
    int t = __builtin_ctzll(m);
    spanv[m] = spanv[m & (m - 1)] ^ gens[t];
  }
  const u64 umask = (u64(1) << u) - 1;
  std::vector<int> send(32), srcl(32), recv(32);
  T.send_slot.assign(T.rounds, 0);
  T.recv_slot.assign(T.rounds, 0);
  T.src_lane0.assign(T.rounds, 0);
  int Mcol[5] = {0}, Kcol[5] = {0}, Ncol[5] = {0};
  for (int r = 0; r < T.rounds; ++r) {
    u64 base = 0;
    for (size_t t = 0; t < T.Rb.size(); ++t) if ((r >> t) & 1) base ^= T.Rb[t];
    std::fill(send.begin(), send.end(), -1);
    std::fill(srcl.begin(), srcl.end(), -1);
    for (u64 s : spanv) {
      u64 x = base ^ s;
      u64 hl = hw_of(invLd, x), hs = hw_of(invSt, x);
      int lane_ld = int((hl >> R) & 31), lane_st = int((hs >> R) & 31);
      int unit_ld = int((hl & ((u64(1) << R) - 1)) >> u);
      int unit_st = int((hs & ((u64(1) << R) - 1)) >> u);
      if ((hl & umask) != (hs & umask)) return false;
      if (send[lane_ld] >= 0 && send[lane_ld] != unit_ld) return false;
      send[lane_ld] = unit_ld;
      if (srcl[lane_st] >= 0 && srcl[lane_st] != lane_ld) return false;
      srcl[lane_st] = lane_ld;
      recv[lane_st] = unit_st;
    }
    for (int l = 0; l < 32; ++l) if (send[l] < 0 || srcl[l] < 0) return false;
    int c, col[5];
    if (!fit_affine(send, c, col)) return false;
    if (r == 0) std::copy(col, col + 5, Mcol);
    else if (!std::equal(col, col + 5, Mcol)) return false;
    T.send_slot[r] = c;
    if (!fit_affine(srcl, c, col)) return false;
    if (r == 0) std::copy(col, col + 5, Kcol);
    else if (!std::equal(col, col + 5, Kcol)) return false;
    T.src_lane0[r] = uint32_t(c);
    if (!fit_affine(recv, c, col)) return false;
    if (r == 0) std::copy(col, col + 5, Ncol);
    else if (!std::equal(col, col + 5, Ncol)) return false;
    T.recv_slot[r] = c;
  }
  for (int t = 0; t < 5; ++t) T.src_lane_col[t] = uint32_t(Kcol[t]);
  xor_network(Mcol, T.pre_lmask, T.pre_x);
  xor_network(Ncol, T.post_lmask, T.post_x);
  // send slots must be a bijection over the rounds (in-place exchange)
  std::vector<int> seen(T.nslot, 0);
  for (int r = 0; r < T.rounds; ++r) if (seen[T.send_slot[r]]++) return false;
  return true;
}

// Shuffles of sub-word elements (w < 4) whose 32-bit unit is not common at the lowest
// register bits (reading R-V): choose the unit V among the logical vectors common to
// both sides' registers (in L_ld's register order), move it to the lowest
// register bits of each side by a thread-local element permutation (prmt / bit-field
// moves — the "prmt.b32 when sub-32-bit elements change position" of row a6), and plan
// the paper's shuffle between the permuted layouts.
static bool plan_shuffle_eperm(TilePlan& T) {
  const int R = T.R, w = T.w;
  if (w >= 4) return false;
  const int u = ilog2(u64(4 / w));
  if (u > R) return false;
  std::vector<int> common;   // L_ld register positions whose column is a register of L_st
  for (int b = 0; b < R; ++b)
    for (int c = 0; c < R; ++c) if (T.lcol_ld[b] == T.lcol_st[c]) common.push_back(b);
  if (int(common.size()) < u) return false;
  const std::vector<u64> ld0 = T.lcol_ld, st0 = T.lcol_st;
  auto reorder = [&](const std::vector<u64>& lc, const std::vector<u64>& V, std::vector<int>& perm_bits) {
    // new register order: V first (in V's order), then the other registers ascending
    std::vector<int> order;
    for (u64 c : V) for (int b = 0; b < R; ++b) if (lc[b] == c) order.push_back(b);
    for (int b = 0; b < R; ++b) if (std::find(order.begin(), order.end(), b) == order.end()) order.push_back(b);
    perm_bits = order;   // new register bit k = old register bit order[k]
    std::vector<u64> out = lc;
    for (int k = 0; k < R; ++k) out[k] = lc[order[k]];
    return out;
  };
  // element e' of the new order = element e of the old order with bit order[k] = bit k of e'
  auto eperm = [&](const std::vector<int>& order) {
    std::vector<int> src(size_t(1) << R);
    for (int e2 = 0; e2 < (1 << R); ++e2) {
      int e = 0;
      for (int k = 0; k < R; ++k) if ((e2 >> k) & 1) e |= 1 << order[k];
      src[e2] = e;
    }
    return src;
  };
  // candidate units: u-subsets of the common vectors, in L_ld's register order
  std::vector<int> pick(u);
  std::function<bool(int, int)> rec = [&](int start, int k) -> bool {
    if (k == u) {
      std::vector<u64> V;
      for (int b : pick) V.push_back(ld0[b]);
      std::vector<int> oa, ob;
      T.lcol_ld = reorder(ld0, V, oa);
      T.lcol_st = reorder(st0, V, ob);
      if (plan_shuffle(T)) {
        T.pre_eperm = eperm(oa);
        // shuffle output (new st order) element e2 holds old-st element eperm(ob)[e2]:
        // the stored element e takes the e2 with eperm(ob)[e2] = e
        const std::vector<int> fwd = eperm(ob);
        T.post_eperm.assign(fwd.size(), 0);
        for (size_t e2 = 0; e2 < fwd.size(); ++e2) T.post_eperm[fwd[e2]] = int(e2);
        T.lcol_ld = ld0;
        T.lcol_st = st0;
        return true;
      }
      return false;
    }
    for (size_t i = start; i < common.size(); ++i) {
      pick[k] = common[i];
      if (rec(int(i) + 1, k + 1)) return true;
    }
    return false;
  };
  const bool ok = rec(0, 0);
  T.lcol_ld = ld0;
  T.lcol_st = st0;
  if (!ok) { T.pre_eperm.clear(); T.post_eperm.clear(); }
  return ok;
}

// Simulated wavefront count (Lemma 9.4 model) of a kernel layout
// accessing smem through offsets `smoff` (per kernel bit) with `v` vector bits.
static long sim_wavefronts(const TilePlan& T, const std::vector<u64>& smoff,
                           const std::vector<int>& vec_slots, long* ideal) {
  const int R = T.R, w = T.w, v = int(vec_slots.size());
  const int a = (1 << v) * w;
  const int lanes_per_phase = a > 4 ? std::max(1, 128 / a) : 32;
  std::vector<int> other;
  for (int b = 0; b < R; ++b)
    if (std::find(vec_slots.begin(), vec_slots.end(), b) == vec_slots.end()) other.push_back(b);
  long total = 0, id = 0;
  for (int wi = 0; wi < (1 << T.Wb); ++wi) {
    u64 wbase = 0;
    for (int t = 0; t < T.Wb; ++t) if ((wi >> t) & 1) wbase ^= smoff[R + 5 + t];
    for (u64 ri = 0; ri < (u64(1) << other.size()); ++ri) {
      u64 rbase = wbase;
      for (size_t t = 0; t < other.size(); ++t) if ((ri >> t) & 1) rbase ^= smoff[other[t]];
      u64 addr[32];
      for (int l = 0; l < 32; ++l) {
        u64 o = rbase;
        for (int t = 0; t < 5; ++t) if ((l >> t) & 1) o ^= smoff[R + t];
        addr[l] = o * w;
      }
      for (int p0 = 0; p0 < 32; p0 += lanes_per_phase) {
        std::map<int, std::vector<u64>> bank;
        for (int l = p0; l < p0 + lanes_per_phase; ++l)
          for (int b = 0; b < a; b += std::min(a, 4)) {
            u64 word = (addr[l] + b) / 4;
            auto& vv = bank[int(word % 32)];
            if (std::find(vv.begin(), vv.end(), word) == vv.end()) vv.push_back(word);
          }
        size_t mx = 0;
        for (auto& kv : bank) mx = std::max(mx, kv.second.size());
        total += long(mx);
        id += (lanes_per_phase * a + 127) / 128;
      }
    }
  }
  if (ideal) *ideal = id;
  return total;
}

// Simulated wavefronts (same model) of a side executed with stmatrix /
// ldmatrix (kind SMI_MAT / SMI_MATT): every 8x8 b16 matrix is 8 rows of 16 bytes
// addressed by 8 lanes, one 128-byte wavefront when the rows fall in distinct
// 16-byte bank groups ("8 groups of 4 threads collaborating to store a row").
static long sim_mat_wavefronts(const TilePlan& T, const std::vector<u64>& smoff, int kind,
                               const std::vector<int>& word, long* ideal) {
  const int R = T.R, w = T.w;
  u64 rows[3];
  for (int t = 0; t < 3; ++t)
    rows[t] = kind == SMI_MAT ? smoff[R + 2 + t] : (t == 0 ? smoff[word[0]] : smoff[R + t - 1]);
  std::vector<u64> other;   // bits enumerating the matrices: non-word registers, warps
  for (int b = 0; b < R; ++b)
    if (std::find(word.begin(), word.end(), b) == word.end()) other.push_back(smoff[b]);
  for (int t = 0; t < T.Wb; ++t) other.push_back(smoff[R + 5 + t]);
  long total = 0, id = 0;
  for (u64 m = 0; m < (u64(1) << other.size()); ++m) {
    u64 base = 0;
    for (size_t t = 0; t < other.size(); ++t) if ((m >> t) & 1) base ^= other[t];
    int cnt[8] = {0};
    for (int r = 0; r < 8; ++r) {
      u64 o = base;
      for (int t = 0; t < 3; ++t) if ((r >> t) & 1) o ^= rows[t];
      ++cnt[(o * u64(w) / 16) % 8];
    }
    total += *std::max_element(cnt, cnt + 8);
    id += 1;
  }
  if (ideal) *ideal = id;
  return total;
}

static void plan_smem(TilePlan& T, int maxvec, int smem_instr) {
  // Optimal swizzling (appendix) on the kernel layouts.
  const int R = T.R, w = T.w, n = T.n;
  auto reg_of = [&](const std::vector<u64>& lc, u64 c) {
    for (int q = 0; q < R; ++q) if (lc[q] == c) return q;
    return -1;
  };
  // 1. Vec: common register vectors, in L_ld register order, within max_vec_bytes
  //    (vectorised ld/st.shared on both sides, tile id_n^{Reg,Off}).
  T.sw_vec.clear(); T.vec_slot_ld.clear(); T.vec_slot_st.clear();
  T.smi_ld = T.smi_st = SMI_VEC;
  T.mat_word_ld.clear(); T.mat_word_st.clear(); T.mat_sel_ld.clear(); T.mat_sel_st.clear();
  for (int b = 0; b < R; ++b) {
    u64 c = T.lcol_ld[b];
    int bs = reg_of(T.lcol_st, c);
    if (bs < 0) continue;
    if ((int(1) << (T.sw_vec.size() + 1)) * w > maxvec) break;
    T.sw_vec.push_back(c);
    T.vec_slot_ld.push_back(b);
    T.vec_slot_st.push_back(bs);
  }
  // 1b. stmatrix / ldmatrix (Thm 5.1).  Their tile makes a 16-byte row of
  //     k = log2(4/w) register bits and lanes 0, 1 (or, transposed, of lanes 2-4), so a
  //     side whose registers share too few vectors with the other side still moves
  //     whole 16-byte rows.  The row is the Vec of the swizzle; M is built with it as
  //     the lowest offset bits, so M^{-1}∘L is divisible by the tile by construction
  //     (the planner asserts it below).  Tried when the common registers give less than
  //     16 bytes (auto) or always (smem_instr = 2); the first divisible choice wins, in
  //     the order: one side matrix, the other vectorised; then both sides matrix.
  const int full = w <= 4 ? ilog2(u64(16 / w)) : 0;
  const int k = w <= 4 ? ilog2(u64(4 / w)) : 0;
  // auto: the matrix tiles are tried when the common registers give less than 16 bytes
  // — under faithful σ less than 8 (measured: its L1-allocating per-thread loads make
  // STSM a net loss when the vectorised path already moves 8 bytes, config 2: 3237 vs
  // 2822 GB/s; a gain from 4 bytes, config 3: 3276 -> 3342; profiles/r01_thm51_*)
  const int want = T.sigma == SIGMA_FAITHFUL ? full - 1 : full;
  if (smem_instr != 1 && w <= 4 && maxvec >= 16 && R >= k &&
      (int(T.sw_vec.size()) < want || smem_instr == 2)) {
    struct Side { int kind; std::vector<int> word; std::vector<u64> row; };
    auto options = [&](const std::vector<u64>& lc) {
      std::vector<Side> out;
      std::vector<std::vector<int>> words;
      if (k == 0) words.push_back({});
      for (int a = 0; a < R && k >= 1; ++a) {
        if (k == 1) { words.push_back({a}); continue; }
        for (int b2 = 0; b2 < R; ++b2) if (b2 != a) words.push_back({a, b2});
      }
      for (auto& wd : words) {
        Side s{SMI_MAT, wd, {}};
        for (int q : wd) s.row.push_back(lc[q]);
        s.row.push_back(lc[R]);
        s.row.push_back(lc[R + 1]);
        out.push_back(s);
      }
      if (w == 2)
        for (auto& wd : words) out.push_back(Side{SMI_MATT, wd, {lc[R + 2], lc[R + 3], lc[R + 4]}});
      return out;
    };
    auto optL = options(T.lcol_ld), optS = options(T.lcol_st);
    auto vec_slots = [&](const std::vector<u64>& lc, const std::vector<u64>& row, std::vector<int>& sl) {
      sl.clear();
      for (u64 c : row) { int q = reg_of(lc, c); if (q < 0) return false; sl.push_back(q); }
      return true;
    };
    bool found = false;
    std::vector<int> sl;
    for (int pass = 0; pass < 3 && !found; ++pass) {
      if (pass == 0)        // matrix stores, vectorised loads
        for (auto& o : optL) {
          if (vec_slots(T.lcol_st, o.row, sl)) {
            T.smi_ld = o.kind; T.mat_word_ld = o.word; T.sw_vec = o.row;
            T.vec_slot_st = sl; T.vec_slot_ld.clear(); found = true; break;
          }
        }
      else if (pass == 1)   // vectorised stores, matrix loads
        for (auto& o : optS) {
          if (vec_slots(T.lcol_ld, o.row, sl)) {
            T.smi_st = o.kind; T.mat_word_st = o.word; T.sw_vec = o.row;
            T.vec_slot_ld = sl; T.vec_slot_st.clear(); found = true; break;
          }
        }
      else
        for (auto& a : optL) {
          for (auto& b : optS)
            if (a.row == b.row) {
              T.smi_ld = a.kind; T.mat_word_ld = a.word; T.smi_st = b.kind; T.mat_word_st = b.word;
              T.sw_vec = a.row; T.vec_slot_ld.clear(); T.vec_slot_st.clear(); found = true; break;
            }
          if (found) break;
        }
    }
    // matrix-select bits: up to two of the remaining registers (.x4)
    auto sel = [&](const std::vector<int>& word, std::vector<int>& s) {
      s.clear();
      for (int b = 0; b < R && s.size() < 2; ++b)
        if (std::find(word.begin(), word.end(), b) == word.end()) s.push_back(b);
    };
    if (T.smi_ld != SMI_VEC) sel(T.mat_word_ld, T.mat_sel_ld);
    if (T.smi_st != SMI_VEC) sel(T.mat_word_st, T.mat_sel_st);
  }
  const int v = int(T.sw_vec.size());
  T.sm_v = v;
  const int vec_bytes = (1 << v) * w;
  // 2. b = log2(128 / (2^v w))
  int b = std::max(0, ilog2(u64(std::max(1, 128 / vec_bytes))));
  if (b > n - v) b = n - v;
  // 3. A_Bank, B_Bank: the vectors enumerating one 128-byte wavefront.  Vectorised
  //    side: its lanes without the last log2 max(1, 2^v w / 4).  Matrix side:
  //    the vectors addressing the 8 rows of one matrix (lanes 2-4; transposed: word
  //    bit, lanes 0, 1).
  int drop = ilog2(u64(std::max(1, vec_bytes / 4)));
  std::vector<u64> aThr(T.lcol_ld.begin() + R, T.lcol_ld.begin() + R + 5);
  std::vector<u64> bThr(T.lcol_st.begin() + R, T.lcol_st.begin() + R + 5);
  auto bank_of = [&](int kind, const std::vector<u64>& lc, const std::vector<int>& word,
                     const std::vector<u64>& thr) {
    if (kind == SMI_MAT) return std::vector<u64>{lc[R + 2], lc[R + 3], lc[R + 4]};
    if (kind == SMI_MATT) return std::vector<u64>{lc[word[0]], lc[R], lc[R + 1]};
    return std::vector<u64>(thr.begin(), thr.end() - drop);
  };
  std::vector<u64> aBank = bank_of(T.smi_ld, T.lcol_ld, T.mat_word_ld, aThr);
  std::vector<u64> bBank = bank_of(T.smi_st, T.lcol_st, T.mat_word_st, bThr);
  // 4. E, F, H
  std::vector<u64> E, F;
  for (u64 c : aBank) if (std::find(bBank.begin(), bBank.end(), c) == bBank.end()) E.push_back(c);
  for (u64 c : bBank) if (std::find(aBank.begin(), aBank.end(), c) == aBank.end()) F.push_back(c);
  if (E.size() > F.size()) std::swap(E, F);
  std::sort(E.begin(), E.end());
  std::sort(F.begin(), F.end());
  T.sw_H.clear();
  for (size_t i = 0; i < E.size(); ++i) T.sw_H.push_back(E[i] ^ F[i]);
  // 5. C completes span(Vec ∪ A_Bank ∪ B_Bank) inside the tile space
  std::vector<u64> space(T.lcol_ld.begin(), T.lcol_ld.end());
  std::sort(space.begin(), space.end());
  Echelon ep;
  for (u64 c : T.sw_vec) ep.insert(c);
  for (u64 c : aBank) ep.insert(c);
  for (u64 c : bBank) ep.insert(c);
  T.sw_C.clear();
  for (u64 c : space) if (ep.insert(c)) T.sw_C.push_back(c);
  // 6. Seg: ℓ vectors from H then C; else unused A_Bank, then A_Thr (G14)
  const int ell = n - v - b;
  Echelon es;
  for (u64 c : T.sw_vec) es.insert(c);
  T.sw_seg.clear();
  auto try_add = [&](u64 c) {
    if (int(T.sw_seg.size()) < ell && es.insert(c)) T.sw_seg.push_back(c);
  };
  for (u64 c : T.sw_H) try_add(c);
  for (u64 c : T.sw_C) try_add(c);
  for (u64 c : aBank) try_add(c);
  for (u64 c : aThr) try_add(c);
  for (u64 c : space) try_add(c);
  // 7. Bank completes span(Vec ∪ Seg)
  T.sw_bank.clear();
  for (u64 c : space) if (es.insert(c)) T.sw_bank.push_back(c);
  if (int(T.sw_vec.size() + T.sw_bank.size() + T.sw_seg.size()) != n)
    fail(LL_ERR_UNSUPPORTED, "swizzle: basis incomplete (internal): |Vec| " + std::to_string(T.sw_vec.size()) +
                                 " |Bank| " + std::to_string(T.sw_bank.size()) + " |Seg| " + std::to_string(T.sw_seg.size()) +
                                 " n " + std::to_string(n));
  // M: offset bit -> logical (Vec, Bank, Seg); invert to get smem offsets.
  std::vector<u64> M = T.sw_vec;
  M.insert(M.end(), T.sw_bank.begin(), T.sw_bank.end());
  M.insert(M.end(), T.sw_seg.begin(), T.sw_seg.end());
  Echelon em;
  for (size_t o = 0; o < M.size(); ++o) em.insert(M[o], u64(1) << o);
  auto minv = [&](u64 x) { u64 c = 0; if (em.reduce(x, &c)) fail(LL_ERR_UNSUPPORTED, "swizzle: not invertible"); return c; };
  T.smoff_ld.resize(n);
  T.smoff_st.resize(n);
  for (int q = 0; q < n; ++q) { T.smoff_ld[q] = minv(T.lcol_ld[q]); T.smoff_st[q] = minv(T.lcol_st[q]); }
  // Thm 5.1: each side's M^{-1}∘L must be divisible by its instruction's tile — the
  // tile's hardware bits are offset bits 0..v-1 in order, and (Def 4.4) no other
  // hardware bit reaches them.
  auto check_tile = [&](int kind, const std::vector<u64>& so, const std::vector<int>& vslot,
                        const std::vector<int>& word) {
    std::vector<int> tile;
    if (kind == SMI_VEC) tile = vslot;
    else if (kind == SMI_MAT) { tile = word; tile.push_back(R); tile.push_back(R + 1); }
    else tile = {R + 2, R + 3, R + 4};
    if (int(tile.size()) != v) fail(LL_ERR_UNSUPPORTED, "swizzle: tile size (internal)");
    const u64 low = (u64(1) << v) - 1;
    for (int q = 0; q < n; ++q) {
      auto it = std::find(tile.begin(), tile.end(), q);
      if (it != tile.end() ? so[q] != (u64(1) << (it - tile.begin())) : (so[q] & low) != 0)
        fail(LL_ERR_UNSUPPORTED, "swizzle: M^-1∘L not divisible by the instruction tile (internal)");
    }
  };
  check_tile(T.smi_ld, T.smoff_ld, T.vec_slot_ld, T.mat_word_ld);
  check_tile(T.smi_st, T.smoff_st, T.vec_slot_st, T.mat_word_st);
  T.smem_elems = u64(1) << n;
  long id1 = 0, id2 = 0;
  T.predicted_wavefronts_st = T.smi_ld == SMI_VEC ? sim_wavefronts(T, T.smoff_ld, T.vec_slot_ld, &id1)
                                                  : sim_mat_wavefronts(T, T.smoff_ld, T.smi_ld, T.mat_word_ld, &id1);
  T.predicted_wavefronts_ld = T.smi_st == SMI_VEC ? sim_wavefronts(T, T.smoff_st, T.vec_slot_st, &id2)
                                                  : sim_mat_wavefronts(T, T.smoff_st, T.smi_st, T.mat_word_st, &id2);
  T.ideal_wavefronts = id1 + id2;
  // shared instructions per thread per tile
  auto ninstr = [&](int kind, const std::vector<int>& word, const std::vector<int>& s) {
    if (kind == SMI_VEC) return long(1) << (R - v);
    return long(1) << (R - int(word.size()) - int(s.size()));
  };
  T.smem_instr_st = ninstr(T.smi_ld, T.mat_word_ld, T.mat_sel_ld);
  T.smem_instr_ld = ninstr(T.smi_st, T.mat_word_st, T.mat_sel_st);
}

static void plan_exchange(ConvPlan& P, const ll_plan_opts* opts);

// ---------------------------------------------------------------------------
static void build_tile(ConvPlan& P, const std::vector<int>& S0, const std::vector<int>& D0,
                       std::vector<int> gridS, std::vector<int> gridD, const ll_plan_opts* opts,
                       bool in_cta, u64 grid_only_src = 0) {
  const Layout &A = P.A, &B = P.B;
  TilePlan& T = P.tile;
  T = TilePlan();
  T.w = P.w;
  int maxvec = default_int(opts, &ll_plan_opts::max_vec_bytes, 16);
  int sigma = opts ? opts->sigma : 0;
  int tile_bytes = default_int(opts, &ll_plan_opts::tile_bytes, 16384);
  std::vector<int> S = S0, D = D0;
  // fold low grid bits into the tile while it is small (common vectors)
  std::vector<int> foldS, foldD;
  // faithful σ: folded bits become kernel warps beside the layout's own (≤ 32 warps)
  const size_t max_fold = (sigma == SIGMA_FAITHFUL && in_cta) ? size_t(std::max(0, 5 - A.in_bits("warp"))) : 64;
  while ((u64(1) << S.size()) * u64(P.w) < u64(tile_bytes) && S.size() < 20 && foldS.size() < max_fold) {
    size_t g = 0;
    while (g < gridS.size() && ((grid_only_src >> gridS[g]) & 1)) ++g;
    if (g == gridS.size()) break;
    foldS.push_back(gridS[g]); foldD.push_back(gridD[g]);
    S.push_back(gridS[g]); D.push_back(gridD[g]);
    gridS.erase(gridS.begin() + g); gridD.erase(gridD.begin() + g);
  }
  std::vector<int> Ss = S, Ds = D;
  std::sort(Ss.begin(), Ss.end());
  std::sort(Ds.begin(), Ds.end());
  if (S.size() < 5) fail(LL_ERR_UNSUPPORTED, "tile smaller than a warp");
  if (sigma == SIGMA_FAITHFUL && in_cta) {
    assign_sigma_faithful(T, A, B, foldS, foldD, maxvec);
  } else {
    std::vector<u64> prefer;
    int pw = A.in_pos("warp");
    for (int k = 0; k < A.in_bits("warp"); ++k) prefer.push_back(A.cols[pw + k]);
    for (int s : foldS) prefer.push_back(A.cols[s]);
    // 256 bytes per thread; cross-CTA tiles (always an smem exchange) keep at least 8
    // warps per CTA (measured: 2 GiB transpose 0.91 -> 1.00 of the copy roofline at
    // 4 -> 8 warps, profiles/r01_sweep_next_rows.jsonl)
    int dflt = 256;
    if (!in_cta) dflt = int(std::max<u64>(u64(P.w), std::min<u64>(256, ((u64(1) << Ss.size()) * u64(P.w)) / 256)));
    // layouts whose own CTA tile is small (grid bits folded in up to tile_bytes): 8
    // warps of 64 bytes per thread rather than 2 warps of 256 — measured +4-11% on the
    // folded 16 KiB tiles (c1 batch, the fp8 operand, 2-byte Fig.-1 tiles), to within
    // 1% of the plain streaming kernel (profiles/r02_sweep_small_cta.jsonl)
    else if (!foldS.empty()) dflt = std::max(P.w, 64);
    int thread_bytes = default_int(opts, &ll_plan_opts::thread_bytes, dflt);
    assign_sigma_coalesced(T, A, B, Ss, Ds, prefer, maxvec, thread_bytes);
  }
  T.grid_src_bit = gridS;
  T.grid_dst_bit = gridD;
  T.lcol_ld.resize(T.n);
  T.lcol_st.resize(T.n);
  for (int b = 0; b < T.n; ++b) { T.lcol_ld[b] = A.cols[T.ld_bit[b]]; T.lcol_st[b] = B.cols[T.st_bit[b]]; }
  plan_exchange(P, opts);
}

// The exchange L_ld -> L_st of a tile plan whose kernel layouts (lcol_ld / lcol_st) are
// set: its class (copy, register permutation, shuffle, smem) and that class's plan.
static void plan_exchange(ConvPlan& P, const ll_plan_opts* opts) {
  TilePlan& T = P.tile;
  const int maxvec = default_int(opts, &ll_plan_opts::max_vec_bytes, 16);
  // exchange class of L_ld -> L_st
  bool same_lane = true, same_warp = true, same_reg = true;
  for (int t = 0; t < 5; ++t) same_lane &= T.lcol_ld[T.R + t] == T.lcol_st[T.R + t];
  for (int t = 0; t < T.Wb; ++t) same_warp &= T.lcol_ld[T.R + 5 + t] == T.lcol_st[T.R + 5 + t];
  for (int t = 0; t < T.R; ++t) same_reg &= T.lcol_ld[t] == T.lcol_st[t];
  int force = opts ? opts->force_class : -1;
  if (force == LL_CLASS_SMEM) {
    T.xchg = X_SMEM;
  } else if (same_lane && same_warp) {
    T.xchg = same_reg ? X_COPY : X_REGPERM;
  } else if (same_warp && plan_shuffle(T)) {
    T.xchg = X_SHUFFLE;
  } else if (same_warp && P.cls <= LL_CLASS_SHUFFLE && plan_shuffle_eperm(T)) {
    // only where the paper's class is SHUFFLE: measured against the smem exchange, the
    // permuted shuffle wins on the fp8 operand conversion (6365 vs 6099 GB/s) and loses
    // where the class is SMEM (config 3b: 5968 vs 6338; profiles/r02_sweep_eperm.jsonl)
    T.xchg = X_SHUFFLE;
  } else {
    if (force == LL_CLASS_SHUFFLE) fail(LL_ERR_UNSUPPORTED, "SHUFFLE forced but the kernel layouts need smem");
    T.xchg = X_SMEM;
  }
  if (T.xchg == X_REGPERM) plan_regperm(T);
  if (T.xchg == X_SMEM) {
    // Tiles of general linear maps (build_linear_tile): the kernel layouts' columns need
    // not be unit vectors, and a wide Vec may leave no complement that every other bit of
    // both sides lies in (M^{-1}∘L not divisible by the instruction tile, Thm 5.1): the
    // vector then narrows until the tile divides (at one element it always does).
    for (int mv = maxvec;; mv /= 2) {
      try {
        plan_smem(T, mv, opts ? opts->smem_instr : 0);
        break;
      } catch (const Error& e) {
        if (mv <= T.w) throw;
      }
    }
  }
  if (T.xchg == X_SMEM) {
    // software-pipelined smem exchange (next tile's loads before this tile's stores):
    // measured slower on every default-sized config — the second register buffer costs
    // occupancy (profiles/r01_sweep_smem_pipeline.jsonl) — so only on request (pipe = 2,
    // LL_PIPE=1).  Linear tiles first took it by default (one CTA per SM: 1.0-1.29x,
    // profiles/r01_sweep_linear_pipe.jsonl); with their addresses kept out of the tile
    // loop (NOHOIST) two unpipelined CTAs per SM measured better on average (mean 0.87 vs
    // 0.82 of copy over six random R2 maps, profiles/r01_sweep_linear_nohoist.jsonl)
    const char* e = std::getenv("LL_PIPE");
    const int op = opts ? opts->pipe : 0;
    T.pipe = e ? std::string(e) == "1" : op == 2;
    // staged (pipe = 3 / LL_PIPE=staged): cp.async double-buffered src stages; needs
    // 16-byte load vectors and room for the exchange buffer plus two raw tiles
    const bool want_staged = e ? std::string(e) == "staged" : op == 3;
    const u64 tile_b = (u64(1) << T.n) * u64(T.w);
    if (want_staged && (T.w << T.vld) == 16 && T.smem_elems * u64(T.w) + 2 * tile_b <= 227 * 1024) {
      T.staged = true;
      T.pipe = false;
    }
    // bulk (pipe = 4 / LL_PIPE=bulk, bulk_st also stores by bulk copy: pipe = 5 /
    // LL_PIPE=bulkst): the CTA tile is contiguous in src-packed order (kernel load bits
    // = the lowest n packed bits), whole tiles by cp.async.bulk into raw stages
    const std::string pe = e ? std::string(e) : "";
    const bool want_bulk = e ? (pe == "bulk" || pe == "bulkst") : (op == 4 || op == 5);
    const bool want_bulk_st = e ? pe == "bulkst" : op == 5;
    auto contiguous = [&](const std::vector<int>& bits) {
      std::vector<int> b = bits;
      std::sort(b.begin(), b.end());
      for (int k = 0; k < int(b.size()); ++k) if (b[k] != k) return false;
      return true;
    };
    if (want_bulk && T.ld_xcol.empty() && !T.staged && contiguous(T.ld_bit) && tile_b <= (u64(1) << 16)) {
      // the dst stage is the exchange buffer itself (read out before it is rewritten)
      const bool st_ok = want_bulk_st && contiguous(T.st_bit) && T.rep_bits.empty() &&
                         (T.w << T.vst) >= 4 && T.smem_elems * u64(T.w) >= tile_b;
      for (int ns = 3; ns >= 2; --ns) {
        const u64 need = T.smem_elems * u64(T.w) + u64(ns) * tile_b + 8 * ns;
        if (need <= 227 * 1024) {
          T.bulk = true;
          T.bulk_st = st_ok;
          T.bulk_stages = ns;
          T.pipe = false;
          break;
        }
      }
    }
  }
  // Resident CTAs per SM (ptxas register cap).  Linear tiles compile to 140-255
  // registers (XOR addresses that cannot fold into immediates), i.e. one CTA per SM;
  // asking for 2 trades registers for a few spills: with NOHOIST 1.07-2.2x over one
  // uncapped CTA on five of six random R2 maps (profiles/r01_sweep_linear_nohoist.jsonl);
  // ll_plan_autotune times both.  Shuffle / smem exchanges with 256 bytes per thread
  // (<= 8 warps): without a minimum-blocks hint ptxas compiles config 3's kernel to 62
  // registers, fewer than the 64 that hold all 16 loads of a thread, so it splits the
  // loads; with __launch_bounds__(threads, 2) it takes 104-110 registers and keeps every
  // load in flight (at most 2 CTAs per SM at 8 warps).  Measured: c3 +1.7%, c3b +4.8%,
  // c2 +0.5%, tcgen05 32x32b / 16x256b +1.4% / +1.7%, 16x64b / 16x128b unchanged
  // (profiles/r02_sweep_smem_occupancy.jsonl, r02_sweep_shuffle_occupancy.jsonl).
  {
    const char* e = std::getenv("LL_MIN_BLOCKS");
    const int om = opts ? opts->min_blocks : 0;
    if (e) T.min_blocks = std::max(0, std::atoi(e));
    else if (om > 0) T.min_blocks = om;
    else if (om == 0 && T.ld_run >= 0 && T.xchg == X_SMEM && !T.staged) T.min_blocks = 2;
    else if (om == 0 && (T.xchg == X_SMEM || T.xchg == X_SHUFFLE) && !T.staged && !T.bulk && !T.pipe &&
             T.Wb <= 3 && (u64(T.w) << T.R) >= 256)
      T.min_blocks = 2;
    else T.min_blocks = 0;
  }
  if (T.xchg == X_SMEM && (T.smem_elems * u64(T.w)) > 200 * 1024)
    fail(LL_ERR_UNSUPPORTED, "smem tile too large");
  P.smem_bytes = T.xchg == X_SMEM ? int(T.smem_elems * T.w) : 0;
  if (T.staged) P.smem_bytes += int(2 * (u64(1) << T.n) * u64(T.w));
  if (T.bulk) P.smem_bytes += int(u64(T.bulk_stages) * (u64(1) << T.n) * u64(T.w) + 8 * T.bulk_stages);
}

// CTA class (Q mixes block/offset bits): choose the dst bits a CTA owns so that both
// the loads and the stores are coalesced.
// grid_only_src: src bits that must stay CTA-index bits (the src dev bits of a peer
// exchange, whose tiles must load from one rank).
static void choose_cta_tile(const std::vector<int>& pi, int nloc, int c_bits,
                            int target_bits, std::vector<int>& S, std::vector<int>& D,
                            std::vector<int>& gS, std::vector<int>& gD, u64 grid_only_src = 0,
                            int c_ld_bits = -1) {
  // dst runs of 2^c_bits elements, src runs of 2^c_ld_bits (default: the same)
  if (c_ld_bits < 0) c_ld_bits = c_bits;
  std::vector<int> inv(nloc, -1);
  for (int k = 0; k < nloc; ++k) inv[pi[k]] = k;
  std::vector<char> inT(nloc, 0);
  auto ok = [&](int d) { return !((grid_only_src >> pi[d]) & 1); };
  for (int k = 0; k < std::min(c_bits, nloc); ++k)
    if (ok(k)) inT[k] = 1;
  for (int k = 0; k < std::min(c_ld_bits, nloc); ++k)
    if (ok(inv[k])) inT[inv[k]] = 1;
  int cnt = 0;
  for (int k = 0; k < nloc; ++k) cnt += inT[k];
  for (int k = 0; k < nloc && cnt < target_bits; ++k) if (!inT[k] && ok(k)) { inT[k] = 1; ++cnt; }
  S.clear(); D.clear(); gS.clear(); gD.clear();
  for (int k = 0; k < nloc; ++k) {
    if (inT[k]) { D.push_back(k); S.push_back(pi[k]); }
    else { gD.push_back(k); gS.push_back(pi[k]); }
  }
}

// General invertible pull maps (memory layouts whose Q scatters the low bits: any Def
// 4.14 layout, Thm 4.13; products of swizzles and transposes).  A CTA tile is
// the dst subspace spanned by a set D of dst bits chosen so that Q(span D) contains the
// low src bits [0, c): loads (XOR-addressed src vectors, LD_XOR) and stores both run
// over contiguous 2^c-element runs, and the exchange between the two kernel layouts is
// planned as for any tile (shuffle / smem with the optimal swizzle).  The logical
// column of a loaded src vector s is A(s).  Returns false when no tile of <= 64 KiB
// exists (the generic kernel then runs).
static bool build_linear_tile(ConvPlan& P, const ll_plan_opts* opts) {
  const Layout &A = P.A, &B = P.B;
  const int w = P.w;
  const int nd = B.d_in() - dev_bits(B);   // local bits (the class is below DEVICE)
  if (A.d_in() - dev_bits(A) != nd || int(P.Q.size()) < nd || !A.injective() || !B.injective() || nd > 40)
    return false;
  Echelon eq;   // Q's columns, to invert Q
  for (int k = 0; k < nd; ++k)
    if (!eq.insert(P.Q[k], u64(1) << k)) return false;
  auto qinv = [&](u64 x) { u64 c = 0; eq.reduce(x, &c); return c; };
  auto alog = [&](u64 s) { u64 x = 0; for (int k = 0; k < nd; ++k) if ((s >> k) & 1) x ^= A.cols[k]; return x; };
  const int maxvec = default_int(opts, &ll_plan_opts::max_vec_bytes, 16);
  const int v = std::max(0, ilog2(u64(std::max(1, maxvec / w))));
  if (v + 5 > nd) return false;
  // tile byte cap: 64 KiB, or ll_plan_opts.tile_bytes when given (32 KiB measured 0.61-1.10x
  // of the 64 KiB tiles on random R2 maps, 128 KiB 0.15-0.96x: an autotune candidate,
  // profiles/r01_sweep_linear_maxtile.jsonl)
  const int tb_cap = opts && opts->tile_bytes > 0 ? std::max(opts->tile_bytes, w << (v + 5)) : 65536;
  const int max_bits = ilog2(u64(tb_cap / w));
  // The tile must hold dst bits [0, cs) (store runs of 2^cs elements) and the preimages of
  // src bits [0, cl) (load runs of 2^cl).  cl = v + 1 still fills whole 32-byte sectors on
  // the load side (two 16-byte lane vectors per sector), so L2 traffic stays algorithmic.
  // Balanced (default): maximise the shorter of the two runs first, then their sum — a
  // closure that only fits at cl = v + 1 with cs = v + 5 often fits 128-byte runs on both
  // sides.  Measured on random R2 layouts of 2^28 elements it is never slower and up to
  // 1.8x faster (0.31 -> 0.57 of copy), and it plans tiles where the widest-store rule
  // found none (profiles/r01_sweep_linear_balance.jsonl).  LL_LINEAR_BALANCE=0: the
  // earlier rule, the widest store runs (cs = v + 5, 512 B per warp instruction) and the
  // longest load runs that then fit.
  const char* bal_env = std::getenv("LL_LINEAR_BALANCE");
  const bool balance = !(bal_env && std::string(bal_env) == "0");
  std::vector<char> inD(nd, 0);
  int cnt = 0, cs_best = -1, cl_best = -1;
  auto closure = [&](int cs, int cl, std::vector<char>& in) {
    std::fill(in.begin(), in.end(), 0);
    for (int k = 0; k < cs; ++k) in[k] = 1;
    for (int k = 0; k < cl; ++k) {
      const u64 y = qinv(u64(1) << k);   // the dst vector whose image is src bit k
      for (int d = 0; d < nd; ++d) if ((y >> d) & 1) in[d] = 1;
    }
    return int(std::count(in.begin(), in.end(), 1));
  };
  {
    std::vector<char> tmp(nd, 0);
    auto better = [&](int cs, int cl) {
      if (cs_best < 0) return true;
      if (!balance) return cs > cs_best || (cs == cs_best && cl > cl_best);
      const int m = std::min(cs, cl), mb = std::min(cs_best, cl_best);
      return m > mb || (m == mb && cs + cl > cs_best + cl_best) || (m == mb && cs + cl == cs_best + cl_best && cs > cs_best);
    };
    for (int cs = v + 5; cs >= (balance ? v + 2 : v + 5); --cs)
      for (int cl = v + 5; cl >= v + 1; --cl) {
        if (!better(cs, cl)) continue;
        const int c = closure(cs, cl, tmp);
        if (c <= max_bits) { cs_best = cs; cl_best = cl; cnt = c; inD = tmp; }
      }
  }
  if (cs_best < 0) return false;
  const int cs = cs_best;
  const int target = std::max(v + 5, ilog2(u64(std::max(1, default_int(opts, &ll_plan_opts::tile_bytes, 16384) / w))));
  for (int k = 0; k < nd && cnt < target; ++k) if (!inD[k]) { inD[k] = 1; ++cnt; }
  TilePlan& T = P.tile;
  T = TilePlan();
  T.w = w;
  T.n = cnt;
  int R = std::max(v, ilog2(u64(std::max(1, default_int(opts, &ll_plan_opts::thread_bytes, 256) / w))));
  T.Wb = std::min(5, std::max(0, T.n - 5 - R));
  T.R = T.n - 5 - T.Wb;
  if (T.R < v) return false;
  T.vld = T.vst = v;
  // store side: the 16-byte vector, then lanes over the next cs - v dst bits (2^cs
  // contiguous elements per warp instruction; 512 bytes at cs = v + 5), the remaining
  // lanes over the lowest other bits of D, then the rest of D: registers low, warps high
  std::vector<int> rest;
  for (int k = cs; k < nd; ++k) if (inD[k]) rest.push_back(k);
  T.st_bit.assign(T.n, -1);
  for (int b = 0; b < v; ++b) T.st_bit[b] = b;
  size_t ri = 0;
  for (int t = 0; t < 5; ++t) T.st_bit[T.R + t] = v + t < cs ? v + t : rest[ri++];
  for (int b = v; b < T.R; ++b) T.st_bit[b] = rest[ri++];
  for (int t = 0; t < T.Wb; ++t) T.st_bit[T.R + 5 + t] = rest[ri++];
  // load side: the src vector and lanes over the low src bits (when in the tile's image),
  // then for every other kernel bit the src vector of the same logical element as the
  // store side (common vectors keep the exchange cheap), else any completing vector
  Echelon es;
  T.ld_xcol.assign(T.n, 0);
  std::vector<char> done(T.n, 0);
  u64 dspan = 0;
  for (int k = 0; k < nd; ++k) if (inD[k]) dspan |= u64(1) << k;
  auto in_image = [&](u64 s) { return (qinv(s) & ~dspan) == 0; };
  for (int b = 0; b < v; ++b) { T.ld_xcol[b] = u64(1) << b; es.insert(T.ld_xcol[b]); done[b] = 1; }
  for (int t = 0; t < 5; ++t) {
    const u64 s = u64(1) << (v + t);
    if (in_image(s) && es.insert(s)) { T.ld_xcol[T.R + t] = s; done[T.R + t] = 1; }
  }
  std::vector<u64> pool;
  for (int k = 0; k < nd; ++k) if (inD[k]) pool.push_back(P.Q[k]);
  std::vector<int> order;
  for (int b = v; b < T.R; ++b) order.push_back(b);
  for (int t = 0; t < 5; ++t) order.push_back(T.R + t);
  for (int t = 0; t < T.Wb; ++t) order.push_back(T.R + 5 + t);
  for (int b : order) {
    if (done[b]) continue;
    u64 s = P.Q[T.st_bit[b]];
    if (!es.insert(s)) {
      s = 0;
      for (u64 q : pool) if (es.insert(q)) { s = q; break; }
      if (!s) return false;
    }
    T.ld_xcol[b] = s;
    done[b] = 1;
  }
  if (es.rank != T.n) return false;
  T.ld_run = v;
  T.st_run = cs;
  while (T.ld_run < v + 5 && T.ld_xcol[T.R + (T.ld_run - v)] == (u64(1) << T.ld_run)) ++T.ld_run;
  T.ld_bit = T.st_bit;   // (unused for the load side: ld_xcol)
  // CTA grid: the dst bits outside D, ascending (concurrent CTAs store neighbouring dst
  // runs; ordering by the src side's bits measured no better, r01_sweep_linear_tiles2.jsonl)
  for (int k = 0; k < nd; ++k)
    if (!inD[k]) {
      T.grid_dst_bit.push_back(k);
      T.grid_src_bit.push_back(k);
      T.grid_src_xcol.push_back(P.Q[k]);
    }
  // a column reaching below the vector needs the in-vector XOR permute, which works on
  // vectors of >= 4 bytes (xor_perm_vec); narrower vectors: not a linear tile
  if ((w << v) < 4) {
    const u64 lowm = (u64(1) << v) - 1;
    for (int b = v; b < T.n; ++b) if (T.ld_xcol[b] & lowm) return false;
    for (u64 c : T.grid_src_xcol) if (c & lowm) return false;
  }
  T.lcol_ld.resize(T.n);
  T.lcol_st.resize(T.n);
  for (int b = 0; b < T.n; ++b) { T.lcol_ld[b] = alog(T.ld_xcol[b]); T.lcol_st[b] = B.cols[T.st_bit[b]]; }
  T.sigma = SIGMA_COALESCED;
  plan_exchange(P, opts);
  P.exec = EXEC_TILE;
  return true;
}

// Broadcast stores in dst order (TilePlan::bcast): used when a zero column of B lies
// among the lowest v + 5 dst bits, where per-thread replica stores would leave holes in
// every vector / warp instruction.  The data tile is written to smem in dst-data order
// (bc_smw) and read back along the store tile U = data bits ∪ those low replica bits,
// replica bits contributing 0 to the smem offset (the broadcast copies are
// the same element).  Higher replica bits stay replica offsets (unrolled / grid).
static void plan_bcast_store(ConvPlan& P, const ll_plan_opts* opts) {
  TilePlan& T = P.tile;
  const Layout& B = P.B;
  const int w = T.w;
  if (T.rep_bits.empty() || w > 4 || !T.ld_xcol.empty()) return;
  const char* e = std::getenv("LL_BCAST");
  if (e && std::string(e) == "0") return;
  const int maxvec = default_int(opts, &ll_plan_opts::max_vec_bytes, 16);
  const int v = std::max(0, ilog2(u64(std::max(1, maxvec / w))));
  std::vector<int> low, high;
  for (int r : T.rep_bits) (r < v + 5 ? low : high).push_back(r);
  if (low.empty()) return;
  std::vector<int> Dt(T.st_bit.begin(), T.st_bit.end());
  std::sort(Dt.begin(), Dt.end());
  std::vector<int> U = Dt;
  U.insert(U.end(), low.begin(), low.end());
  std::sort(U.begin(), U.end());
  const int nU = int(U.size());
  if (nU < v + 5 + T.Wb) return;
  for (int i = 0; i < v + 5; ++i) if (U[i] != i) return;   // whole vectors and 512-byte warp runs
  if (nU - v - 5 - T.Wb > 10) return;                       // per-thread vectors (code size)
  auto posD = [&](int k) { return int(std::lower_bound(Dt.begin(), Dt.end(), k) - Dt.begin()); };
  T.bc_smw.assign(T.n, 0);
  for (int b = 0; b < T.n; ++b) {
    int k = -1;
    for (int d : Dt) if (B.cols[d] == T.lcol_ld[b]) k = d;
    if (k < 0) return;                                       // not a data bit of this tile
    T.bc_smw[b] = u64(1) << posD(k);
  }
  T.bc_smr.assign(nU, 0);
  for (int u = 0; u < nU; ++u)
    if (std::binary_search(Dt.begin(), Dt.end(), U[u])) T.bc_smr[u] = u64(1) << posD(U[u]);
  T.bc_U = U;
  T.bc_v = v;
  T.bcast = true;
  T.rep_bits = high;
  T.staged = T.bulk = T.bulk_st = T.pipe = false;
  P.smem_bytes = int((u64(1) << T.n) * u64(w));
}

std::unique_ptr<ConvPlan> plan_convert(const Layout& A, const Layout& B, int w, const ll_plan_opts* opts,
                                       u64 grid_only_src) {
  if (w != 1 && w != 2 && w != 4 && w != 8) fail(LL_ERR_INVALID_ARG, "elem_bytes must be 1, 2, 4 or 8");
  if (A.out != B.out) fail(LL_ERR_DIM_MISMATCH, "A and B must have the same output dims");
  for (auto* L : {&A, &B}) {
    for (auto& d : L->in)
      if (dim_level(d.name) < 0) fail(LL_ERR_INVALID_ARG, "unknown input dim name '" + d.name + "'");
    if (L->d_in() > 62) fail(LL_ERR_INVALID_ARG, "more than 62 input bits");
    int pd = L->in_pos("dev");
    if (pd >= 0 && pd + L->in_bits("dev") != L->d_in()) fail(LL_ERR_INVALID_ARG, "dev must be the last input dim");
  }
  if (!A.surjective()) fail(LL_ERR_NOT_SURJECTIVE, "A is not surjective (Def 4.5, P:194)");
  auto P = std::make_unique<ConvPlan>();
  P->A = A; P->B = B; P->w = w;
  int lev = classify_and_adjust(A, B, P->Q);
  bool noop = A.in == B.in && A.cols == B.cols;
  P->cls = noop ? LL_CLASS_NOOP : ll_class(LL_CLASS_REGPERM + lev);
  const int dA = dev_bits(A), dB = dev_bits(B);
  const int nA = A.d_in() - dA, nB = B.d_in() - dB;
  P->src_elems = u64(1) << nA;
  P->dst_elems = u64(1) << nB;
  P->dev_bits = std::max(dA, dB);
  if (noop) { P->exec = EXEC_NOOP; return P; }
  if (P->cls == LL_CLASS_DEVICE) {
    P->exec = EXEC_DEVICE;
    return P;   // completed by plan_device (dist.cpp)
  }
  // local pull map: dst local bit -> src local index (no dev components by class)
  bool generic = opts && opts->generic;
  bool perm = A.unit_columns() && B.unit_columns() && nA == nB;
  if (!generic && perm) {
    std::vector<int> pi(nB);
    for (int k = 0; k < nB; ++k) {
      u64 q = P->Q[k];
      if (popc(q) != 1 || lead(q) >= nA) { perm = false; break; }
      pi[k] = lead(q);
    }
    if (perm) {
      try {
        std::vector<int> S, D, gS, gD;
        if (lev <= 2 && !grid_only_src) {
          D = bits_at_level(B, 0, 2);
          for (int k : D) S.push_back(pi[k]);
          for (int k : bits_at_level(B, 3, 3)) { gD.push_back(k); gS.push_back(pi[k]); }
          build_tile(*P, S, D, gS, gD, opts, true);
        } else {
          int maxvec = default_int(opts, &ll_plan_opts::max_vec_bytes, 16);
          int v = std::max(0, ilog2(u64(std::max(1, maxvec / w))));
          int tb = default_int(opts, &ll_plan_opts::tile_bytes, 16384);
          int target = std::max(v + 5, ilog2(u64(std::max(1, tb / w))));
          // the longest contiguous runs (2^c elements on both sides) whose tile fits in
          // 64 KiB of smem (or ll_plan_opts.tile_bytes when larger): 512-byte runs, else
          // 256, else 128 (one line)
          const int max_bits = ilog2(u64(std::max(65536, tb) / w));
          // experiment hook LL_CTA_RUNS=<ld extra bits>: src runs longer than the dst runs
          const char* re = std::getenv("LL_CTA_RUNS");
          const int ld_extra = re ? std::atoi(re) : 0;
          for (int c_bits = v + 5; c_bits >= v + 3; --c_bits) {
            choose_cta_tile(pi, nB, c_bits, target, S, D, gS, gD, grid_only_src,
                            ld_extra ? std::min(std::max(c_bits + ld_extra, v + 3), v + 6) : -1);
            if (int(S.size()) <= max_bits) break;
          }
          build_tile(*P, S, D, gS, gD, opts, false, grid_only_src);
        }
        P->exec = EXEC_TILE;
        return P;
      } catch (const Error& e) {
        if (opts && opts->force_class >= 0) throw;
        // fall through to the generic kernel
      }
    }
  }
  // Broadcast layouts (zero columns, rule (2) P:362) inside one CTA: the
  // non-zero columns of A and of B are each a permutation of the logical unit vectors.
  // The kernel moves the distinct elements only: src bits with zero columns are never
  // read (slack = 0), dst bits with zero columns become store replicas.
  auto try_bcast = [&]() -> bool {
    if (generic || lev > 3 || (opts && opts->sigma == SIGMA_FAITHFUL)) return false;
    auto nz_unit = [](const Layout& L) {
      u64 seen = 0;
      for (u64 c : L.cols) {
        if (!c) continue;
        if (popc(c) != 1 || (seen & c)) return false;
        seen |= c;
      }
      return popc(seen) == L.d_out();
    };
    if (nz_unit(A) && nz_unit(B)) {
      try {
        std::vector<int> S, D, gS, gD, rep;
        auto srcbit_of = [&](u64 c) {
          for (int k = 0; k < nA; ++k) if (A.cols[k] == c) return k;
          fail(LL_ERR_UNSUPPORTED, "broadcast: column missing in A (internal)");
        };
        if (lev <= 2) {
          for (int k : bits_at_level(B, 0, 2)) {
            if (B.cols[k]) { D.push_back(k); S.push_back(srcbit_of(B.cols[k])); }
            else rep.push_back(k);
          }
          for (int k : bits_at_level(B, 3, 3)) {
            if (B.cols[k]) { gD.push_back(k); gS.push_back(srcbit_of(B.cols[k])); }
            else rep.push_back(k);
          }
          build_tile(*P, S, D, gS, gD, opts, true);
        } else {
          // CTA class (the map mixes block / offset bits): the data bits of B and the
          // non-zero bits of A form a bit permutation; the CTA tile is chosen on it as in
          // the permutation path (choose_cta_tile), over the data bits
          // compressed to consecutive indices, then mapped back to packed bits
          std::vector<int> Dall, Sall;
          for (int k = 0; k < nB; ++k) (B.cols[k] ? Dall : rep).push_back(k);
          for (int k = 0; k < nA; ++k) if (A.cols[k]) Sall.push_back(k);
          if (Dall.size() != Sall.size()) fail(LL_ERR_UNSUPPORTED, "broadcast: data bits differ (internal)");
          const int nd = int(Dall.size());
          std::vector<int> pi(nd);
          for (int c = 0; c < nd; ++c) {
            const int sb = srcbit_of(B.cols[Dall[c]]);
            pi[c] = int(std::lower_bound(Sall.begin(), Sall.end(), sb) - Sall.begin());
          }
          const int maxvec = default_int(opts, &ll_plan_opts::max_vec_bytes, 16);
          const int v = std::max(0, ilog2(u64(std::max(1, maxvec / w))));
          const int tbytes = default_int(opts, &ll_plan_opts::tile_bytes, 16384);
          const int target = std::max(v + 5, ilog2(u64(std::max(1, tbytes / w))));
          const int max_bits = ilog2(u64(65536 / w));
          std::vector<int> Sc, Dc, gSc, gDc;
          for (int c_bits = v + 5; c_bits >= v + 3; --c_bits) {
            choose_cta_tile(pi, nd, c_bits, target, Sc, Dc, gSc, gDc);
            if (int(Sc.size()) <= max_bits) break;
          }
          for (int c : Sc) S.push_back(Sall[c]);
          for (int c : Dc) D.push_back(Dall[c]);
          for (int c : gSc) gS.push_back(Sall[c]);
          for (int c : gDc) gD.push_back(Dall[c]);
          build_tile(*P, S, D, gS, gD, opts, false);
        }
        P->tile.rep_bits = rep;
        if (!rep.empty()) {
          // replicas: per-thread stores, plain tile loop (no staged / bulk variants);
          // dst-order broadcast stores when a replica bit is low (plan_bcast_store); at
          // most 2 unrolled replica bits, the rest CTA-grid bits below the data tiles'
          // while the grid keeps >= 8 CTAs per SM
          TilePlan& T = P->tile;
          if (T.staged || T.bulk) {
            P->smem_bytes = int(T.smem_elems * u64(T.w));
            T.staged = T.bulk = T.bulk_st = false;
          }
          plan_bcast_store(*P, opts);
          const int nrep = int(T.rep_bits.size());
          const int gdata = int(T.grid_dst_bit.size());
          // measured (profiles/r02_sweep_broadcast_*.jsonl): plans unrolling 16 replicas
          // per store (rep_lo = 4) were the slowest; with the replica group as the low
          // CTA-index bits (the src tile's re-reads hit L2) at most 2 are unrolled
          T.rep_lo = std::min(2, nrep);
          while (T.rep_lo > 0 && (gdata + nrep - T.rep_lo) < 64 && (u64(1) << (gdata + nrep - T.rep_lo)) < u64(8 * 148))
            --T.rep_lo;
        }
        P->exec = EXEC_TILE;
        return true;
      } catch (const Error& e) {
        if (opts && opts->force_class >= 0) throw;
        P->tile = TilePlan();
      }
    }
    return false;
  };
  // lev <= 2: inside one CTA.  CTA class (lev 3): after the XOR-copy tiles below, which
  // keep the widest global vectors on the small memory <-> distributed maps of Table 3
  // (LL_BCAST_CTA=1 tries the CTA-tiled broadcast first, =0 never)
  const char* bce = std::getenv("LL_BCAST_CTA");
  const bool bcast_cta_first = bce && std::string(bce) == "1";
  const bool bcast_cta_never = bce && std::string(bce) == "0";
  if ((lev <= 2 || bcast_cta_first) && try_bcast()) return P;
  // Any other linear pull map (2-bit columns of swizzled memory layouts, Def 4.14 /
  // P:240-276; broadcast across CTAs): a copy kernel in dst order — coalesced 16-byte
  // stores, loads at src = Q(dst) (XOR of columns), vectorised over the low dst bits Q
  // keeps in place.  Efficient when Q is row-local (swizzles); the generic kernel is
  // kept for maps that scatter the low bits.
  if (!generic && lev <= 3 && nB >= 5) {
    int vmax = std::max(0, ilog2(u64(std::max(1, default_int(opts, &ll_plan_opts::max_vec_bytes, 16) / w))));
    // vector bits: dst bits [0, v) map to src bits [0, v), and no other column reaches
    // below bit v, so each vector's 2^v elements are contiguous and aligned in src
    int v = 0;
    while (v < vmax && v < nB && P->Q[v] == (u64(1) << v)) ++v;
    // Other columns may reach below bit v (a swizzle that XORs inside the vector, e.g.
    // Def 4.11 with vec < 16 bytes): each dst vector's elements are then one aligned src
    // vector, permuted by an element XOR — loaded whole and permuted in registers
    // (in-vector XOR, vectors of >= 4 bytes; LL_XOR_INVEC=0 disables).  Otherwise the
    // vector shrinks until no column reaches below it.
    const char* ie = std::getenv("LL_XOR_INVEC");
    const bool invec = !(ie && std::string(ie) == "0") && (w << v) >= 4;
    for (;;) {
      bool clean = true;
      for (int k = v; k < nB; ++k) if (P->Q[k] & ((u64(1) << v) - 1)) clean = false;
      if (clean || v == 0 || invec) break;
      --v;
    }
    const u64 lowm = (u64(1) << v) - 1;
    // the low lane bits must keep whole 32-byte sectors together: Q maps dst bits [v, v+2)
    // to src bits of single weight above the vector
    bool rowlocal = true;
    for (int k = v; k < std::min(nB, v + 2); ++k) if (popc(P->Q[k] & ~lowm) != 1) rowlocal = false;
    if (rowlocal) {
      TilePlan& T = P->tile;
      T = TilePlan();
      T.w = w;
      const int tb = default_int(opts, &ll_plan_opts::tile_bytes, 16384);
      int n = std::min(nB, std::max(v + 5, ilog2(u64(std::max(1, tb / w)))));
      int thread_bytes = default_int(opts, &ll_plan_opts::thread_bytes, 64);
      int R = std::max(v, ilog2(u64(std::max(1, thread_bytes / w))));
      int Wb = std::min(5, std::max(0, n - 5 - R));
      R = n - 5 - Wb;
      if (R >= v) {
        T.n = n; T.R = R; T.Wb = Wb;
        T.vld = T.vst = v;
        // dst bits in order: kreg[0,v), klane, kreg[v,R), kwarp; grid = the top bits
        std::vector<int> order;
        for (int k = 0; k < v; ++k) order.push_back(k);
        std::vector<int> lane_bits, reg_bits, warp_bits;
        int k = v;
        for (int t = 0; t < 5; ++t) lane_bits.push_back(k++);
        for (int t = v; t < R; ++t) reg_bits.push_back(k++);
        for (int t = 0; t < Wb; ++t) warp_bits.push_back(k++);
        T.st_bit = order;
        T.st_bit.insert(T.st_bit.end(), reg_bits.begin(), reg_bits.end());
        T.st_bit.insert(T.st_bit.end(), lane_bits.begin(), lane_bits.end());
        T.st_bit.insert(T.st_bit.end(), warp_bits.begin(), warp_bits.end());
        T.ld_bit = T.st_bit;   // (unused for the load side: ld_xcol)
        for (int b : T.st_bit) T.ld_xcol.push_back(P->Q[b]);
        for (int g = n; g < nB; ++g) {
          T.grid_dst_bit.push_back(g);
          T.grid_src_bit.push_back(g);
          T.grid_src_xcol.push_back(P->Q[g]);
        }
        T.lcol_ld.assign(n, 0);
        T.lcol_st.assign(n, 0);
        for (int b = 0; b < n; ++b) T.lcol_st[b] = T.lcol_ld[b] = B.cols[T.st_bit[b]];
        T.xchg = X_COPY;
        T.sigma = SIGMA_COALESCED;
        P->smem_bytes = 0;
        P->exec = EXEC_TILE;
        return P;
      }
    }
  }
  if (lev == 3 && !bcast_cta_first && !bcast_cta_never && try_bcast()) return P;
  if (!generic && lev <= 3) {
    try {
      if (build_linear_tile(*P, opts)) return P;
    } catch (const Error& e) {
      if (opts && opts->force_class >= 0) throw;
    }
  }
  P->tile = TilePlan();
  P->exec = EXEC_GENERIC;
  return P;
}

// ---------------------------------------------------------------- describe
static std::string vec_json(const std::vector<u64>& v) {
  std::ostringstream o;
  o << "[";
  for (size_t i = 0; i < v.size(); ++i) o << (i ? "," : "") << v[i];
  o << "]";
  return o.str();
}
template <class T>
static std::string ivec_json(const std::vector<T>& v) {
  std::ostringstream o;
  o << "[";
  for (size_t i = 0; i < v.size(); ++i) o << (i ? "," : "") << v[i];
  o << "]";
  return o.str();
}

static std::string smem_instr_name(int kind, bool store, size_t nsel, int v, int w) {
  std::ostringstream o;
  if (kind == SMI_VEC) {
    const int bytes = (1 << v) * w;
    o << (store ? "st" : "ld") << ".shared";
    if (bytes > 4) o << ".v" << bytes / 4 << ".b32";
    else o << ".b" << bytes * 8;
  } else {
    o << (store ? "stmatrix" : "ldmatrix") << ".m8n8.x" << (1 << nsel) << (kind == SMI_MATT ? ".trans" : "") << ".b16";
  }
  return o.str();
}

std::string describe(const ConvPlan& P) {
  static const char* cls[] = {"NOOP", "REGPERM", "SHUFFLE", "SMEM", "CTA", "DEVICE"};
  static const char* ex[] = {"noop", "tile", "generic", "device"};
  static const char* xc[] = {"copy", "regperm", "shuffle", "smem"};
  std::ostringstream o;
  o << "{\"class\":\"" << cls[P.cls] << "\",\"exec\":\"" << ex[P.exec] << "\",\"elem_bytes\":" << P.w
    << ",\"src_elems\":" << P.src_elems << ",\"dst_elems\":" << P.dst_elems
    << ",\"Q\":" << vec_json(P.Q);
  if (P.exec == EXEC_TILE) {
    const TilePlan& T = P.tile;
    o << ",\"tile\":{\"xchg\":\"" << xc[T.xchg] << "\",\"sigma\":\"" << (T.sigma ? "faithful" : "coalesced")
      << "\",\"n\":" << T.n << ",\"R\":" << T.R << ",\"warp_bits\":" << T.Wb << ",\"threads\":" << T.threads()
      << ",\"vld\":" << T.vld << ",\"vst\":" << T.vst << ",\"ctas\":" << (u64(1) << T.grid_dst_bit.size())
      << ",\"ld_bit\":" << ivec_json(T.ld_bit) << ",\"st_bit\":" << ivec_json(T.st_bit)
      << ",\"L_ld\":" << vec_json(T.lcol_ld) << ",\"L_st\":" << vec_json(T.lcol_st)
      << ",\"grid_src_bit\":" << ivec_json(T.grid_src_bit) << ",\"grid_dst_bit\":" << ivec_json(T.grid_dst_bit)
      << ",\"rep_bits\":" << ivec_json(T.rep_bits) << ",\"rep_unrolled\":" << std::min<size_t>(size_t(T.rep_lo), T.rep_bits.size())
      << ",\"bcast_store\":" << (T.bcast ? "true" : "false");
    if (T.bcast) o << ",\"bcast_U\":" << ivec_json(T.bc_U) << ",\"bcast_v\":" << T.bc_v;
    if (!T.ld_xcol.empty())
      o << ",\"ld_xcol\":" << vec_json(T.ld_xcol) << ",\"linear_tile\":" << (T.ld_run >= 0 ? "true" : "false")
        << ",\"ld_run_bits\":" << (T.ld_run >= 0 ? T.ld_run : T.vld + 5)
        << ",\"st_run_bits\":" << (T.st_run >= 0 ? T.st_run : T.vst + 5);
    if (T.xchg == X_SHUFFLE)
      o << ",\"V\":" << vec_json(T.V) << ",\"I\":" << vec_json(T.I) << ",\"E\":" << vec_json(T.E)
        << ",\"F\":" << vec_json(T.F) << ",\"G\":" << vec_json(T.G) << ",\"R_basis\":" << vec_json(T.Rb)
        << ",\"rounds\":" << T.rounds << ",\"pre_stages\":" << T.pre_x.size()
        << ",\"post_stages\":" << T.post_x.size() << ",\"unit_elems\":" << T.unit_elems
        << ",\"element_permutes\":" << (T.pre_eperm.empty() ? "false" : "true")
        << ",\"min_blocks\":" << T.min_blocks;
    if (T.xchg == X_SMEM)
      o << ",\"Vec\":" << vec_json(T.sw_vec) << ",\"Bank\":" << vec_json(T.sw_bank) << ",\"Seg\":" << vec_json(T.sw_seg)
        << ",\"H\":" << vec_json(T.sw_H) << ",\"C\":" << vec_json(T.sw_C)
        << ",\"smem_bytes\":" << T.smem_elems * T.w << ",\"pipe\":" << (T.pipe ? "true" : "false") << ",\"staged\":" << (T.staged ? "true" : "false") << ",\"bulk\":" << (T.bulk ? (T.bulk_st ? "\"load+store\"" : "\"load\"") : "false") << ",\"min_blocks\":" << T.min_blocks
        << ",\"wavefronts_st\":" << T.predicted_wavefronts_st << ",\"wavefronts_ld\":" << T.predicted_wavefronts_ld
        << ",\"ideal_wavefronts\":" << T.ideal_wavefronts
        << ",\"smem_store\":\"" << smem_instr_name(T.smi_ld, true, T.mat_sel_ld.size(), T.sm_v, T.w) << "\""
        << ",\"smem_load\":\"" << smem_instr_name(T.smi_st, false, T.mat_sel_st.size(), T.sm_v, T.w) << "\""
        << ",\"smem_store_instrs\":" << T.smem_instr_st << ",\"smem_load_instrs\":" << T.smem_instr_ld
        << ",\"mat_word_ld\":" << ivec_json(T.mat_word_ld) << ",\"mat_sel_ld\":" << ivec_json(T.mat_sel_ld)
        << ",\"mat_word_st\":" << ivec_json(T.mat_word_st) << ",\"mat_sel_st\":" << ivec_json(T.mat_sel_st)
        << ",\"smoff_ld\":" << vec_json(T.smoff_ld) << ",\"smoff_st\":" << vec_json(T.smoff_st);
    o << "}";
  }
  if (!P.tune_json.empty()) o << ",\"autotune\":" << P.tune_json;
  if (P.exec == EXEC_DEVICE) {
    o << ",\"dev_bits\":" << P.dev_bits << ",\"workspace_bytes\":" << P.workspace_bytes
      << ",\"exchange\":\"" << (P.exchange == LL_EXCHANGE_PEER ? "peer" : "collective") << "\"";
    if (P.fused)
      o << ",\"rank_tiles\":" << P.rank_tiles << ",\"peer_reg\":" << (P.fused->peer_reg ? "true" : "false")
        << ",\"fused\":" << describe(*P.fused);
    if (P.pack) o << ",\"pack\":" << describe(*P.pack);
    if (P.unpack) o << ",\"unpack\":" << describe(*P.unpack);
  }
  o << "}";
  return o.str();
}

// ---------------------------------------------------------------------------
// Gather (§5.5)
// ---------------------------------------------------------------------------
// Line-coalesced kernel decomposition for the single-layout kernels (gather, reduce;
// DESIGN.md §5.6-5.7).  Tile bits (reg, lane, warp of L) in packed order t0 < t1 < ...:
//   kreg[0, v)  = the v lowest reg/lane bits (one 16-byte vector per thread),
//   klane[0, 3) = the next 3 bits (8 lanes cover one 128-byte line),
//   klane[3, 5) = two of the remaining reg/lane bits, those with pref(bit) = true
//                 first, then ascending,
//   kreg[v, R)  = the remaining reg/lane bits ascending,
//   kernel warps = L's warp bits.
static std::vector<int> sigma_line(const Layout& L, int v, const std::function<bool(int)>& pref) {
  auto regb = bits_at_level(L, 0, 0), laneb = bits_at_level(L, 1, 1), warpb = bits_at_level(L, 2, 2);
  const int R = int(regb.size());
  std::vector<int> nw = regb;
  nw.insert(nw.end(), laneb.begin(), laneb.end());
  std::sort(nw.begin(), nw.end());
  if (R < v || int(nw.size()) != R + 5) fail(LL_ERR_UNSUPPORTED, "line σ: bad tile");
  std::vector<int> hw(R + 5 + warpb.size());
  for (int b = 0; b < v; ++b) hw[b] = nw[b];
  for (int t = 0; t < 3; ++t) hw[R + t] = nw[v + t];
  std::vector<int> rest(nw.begin() + v + 3, nw.end());
  std::stable_sort(rest.begin(), rest.end(), [&](int a, int b) { return pref(a) && !pref(b); });
  hw[R + 3] = rest[0];
  hw[R + 4] = rest[1];
  std::vector<int> regs(rest.begin() + 2, rest.end());
  std::sort(regs.begin(), regs.end());
  for (int b = v; b < R; ++b) hw[b] = regs[b - v];
  for (size_t t = 0; t < warpb.size(); ++t) hw[R + 5 + t] = warpb[t];
  return hw;
}

// More warps per CTA for the single-layout kernels (reduce, scan): a register bit of the
// kernel layout that carries no in-tile axis bit (independent rows) becomes an extra warp
// bit, so the CTA tile (the same packed bits: TMA staging unchanged) runs on twice the
// warps with half the registers each — latency hiding for the dependent add / shuffle
// chains.  `thread_bytes` (ll_plan_opts) is the register budget per thread; the vector
// bits [0, v) stay registers, at most 5 warp bits (1024 threads).  Only bits with a
// non-zero, non-axis column move: a zero (broadcast) column stays a dead register rather
// than duplicating whole warps.
static void widen_warps(std::vector<int>& hw_bit, int& R, int& Wb, int v, int thread_bytes,
                        const std::function<bool(int)>& movable) {
  const int Rt = std::max(v, ilog2(u64(std::max(4, thread_bytes) / 4)));
  while (R > Rt && Wb < 5) {
    int b = -1;
    for (int q = R - 1; q >= v; --q) if (movable(hw_bit[q])) { b = q; break; }
    if (b < 0) break;
    const int pk = hw_bit[b];
    hw_bit.erase(hw_bit.begin() + b);
    hw_bit.push_back(pk);   // after the lanes and the existing warps: the new top warp bit
    --R;
    ++Wb;
  }
}

// The reverse step for the grid: while the CTA tile (register, lane and warp bits of the
// kernel layout, 2^(R+5+Wb) elements of w bytes) exceeds `tile_bytes`, its top warp bit
// that carries a non-zero, non-axis column (independent rows: no step of the gather,
// reduction or scan crosses it) becomes a CTA-grid bit.  The CTA tile shrinks, the CTA
// count grows, registers per thread stay.  Returns the moved layout bits in ascending
// packed position: the caller puts them below the layout's block bits, so consecutive
// CTAs cover neighbouring pieces of one layout tile.  0 = keep the layout's CTA tile.
static std::vector<int> split_tile(std::vector<int>& hw_bit, int R, int& Wb, int w, int tile_bytes,
                                   const std::function<bool(int)>& movable) {
  std::vector<int> moved;
  if (tile_bytes <= 0) return moved;
  const int target = std::max(R + 5, ilog2(u64(std::max(1, tile_bytes / w))));
  while (R + 5 + Wb > target && Wb > 0) {
    int q = -1;
    for (int b = int(hw_bit.size()) - 1; b >= R + 5; --b) if (movable(hw_bit[b])) { q = b; break; }
    if (q < 0) break;
    moved.push_back(hw_bit[q]);
    hw_bit.erase(hw_bit.begin() + q);
    --Wb;
  }
  std::sort(moved.begin(), moved.end());
  return moved;
}

std::unique_ptr<GatherPlan> plan_gather(const Layout& L, int axis, int w, const ll_plan_opts* opts) {
  if (w != 1 && w != 2 && w != 4 && w != 8) fail(LL_ERR_INVALID_ARG, "elem_bytes must be 1, 2, 4 or 8");
  if (axis < 0 || axis >= int(L.out.size())) fail(LL_ERR_INVALID_ARG, "axis out of range");
  if (!L.unit_columns()) fail(LL_ERR_UNSUPPORTED, "gather: L must be a bijective distributed layout");
  if (L.in_bits("lane") != 5) fail(LL_ERR_UNSUPPORTED, "gather: 5 lane bits required");
  auto G = std::make_unique<GatherPlan>();
  G->L = L; G->axis = axis; G->w = w;
  const int sh = L.out_shift(axis), ab = L.out[axis].bits;
  const u64 amask = ((ab >= 64) ? ~u64(0) : ((u64(1) << ab) - 1)) << sh;
  auto tileb = bits_at_level(L, 0, 2);
  auto blk = bits_at_level(L, 3, 3);
  // in-tile axis bits must be the low K bits of the axis coordinate (O10)
  std::vector<int> axis_bits;
  for (int k : tileb) if (L.cols[k] & amask) axis_bits.push_back(k);
  G->K_bits = int(axis_bits.size());
  for (int t = 0; t < G->K_bits; ++t) {
    bool found = false;
    for (int k : axis_bits) if (L.cols[k] == (u64(1) << (sh + t))) found = true;
    if (!found) fail(LL_ERR_UNSUPPORTED, "gather: in-tile axis bits must be the low axis bits");
  }
  // the paper's shuffle gather needs L_Wrp^axis = 0; the shared-memory gather
  // stages the whole CTA tile and serves axis bits on any level
  bool warp_axis = false;
  for (int k : bits_at_level(L, 2, 2))
    if (L.cols[k] & amask) warp_axis = true;
  // kernel decomposition: faithful (L itself) or coalesced σ; pick the one with
  // fewer shuffle candidates 2^{|L_Reg^axis|}, coalesced on ties.
  const int ev = std::max(w, 4);   // idx is int32: one σ for both
  int maxvec = default_int(opts, &ll_plan_opts::max_vec_bytes, 16);
  int v = std::min(ilog2(u64(std::max(1, maxvec / ev))), L.in_bits("reg"));
  auto regb = bits_at_level(L, 0, 0), laneb = bits_at_level(L, 1, 1), warpb = bits_at_level(L, 2, 2);
  int R = int(regb.size());

  std::vector<int> faith;
  for (int k : regb) faith.push_back(k);
  for (int k : laneb) faith.push_back(k);
  for (int k : warpb) faith.push_back(k);
  // coalesced (line σ with the axis bits preferred in the free lanes, so that fewer
  // candidates remain in registers) unless faithful is requested: measured on B200,
  // coalesced loads beat faithful ones even at 2x the shuffles (profiles/r01_*).
  std::vector<int> coal = sigma_line(L, v, [&](int k) { return (L.cols[k] & amask) != 0; });
  int sigma = opts ? opts->sigma : 0;
  bool use_coal = sigma != SIGMA_FAITHFUL;
  G->hw_bit = use_coal ? coal : faith;
  G->sigma = use_coal ? SIGMA_COALESCED : SIGMA_FAITHFUL;
  G->R = R;
  G->Wb = int(warpb.size());
  G->v = use_coal ? v : std::min(ilog2(u64(std::max(1, maxvec / ev))), R);
  // extra warps from non-axis register bits (ll_plan_opts.thread_bytes, default 32 bytes
  // of data per thread): measured over the config-4 gathers and Table 4 families x 3 tile
  // shapes at 64 MiB and 1 GiB (profiles/r02_sweep_gather_families.jsonl), direct loads
  // with 32 bytes per thread are within 3% of the best of 24 variants on every case and
  // +5-24% over the former default (the layout's own warps and TMA stages)
  {
    const int tb = default_int(opts, &ll_plan_opts::thread_bytes, 32);
    widen_warps(G->hw_bit, G->R, G->Wb, G->v, tb / w * 4,
                [&](int k) { return L.cols[k] != 0 && (L.cols[k] & amask) == 0; });
    R = G->R;
  }
  // optional smaller CTA tiles (ll_plan_opts.tile_bytes): independent rows to the grid
  const auto gmoved = split_tile(G->hw_bit, G->R, G->Wb, w, opts ? opts->tile_bytes : 0,
                                 [&](int k) { return L.cols[k] != 0 && (L.cols[k] & amask) == 0; });
  G->grid_bit = gmoved;
  G->grid_bit.insert(G->grid_bit.end(), blk.begin(), blk.end());
  G->lcol.resize(G->hw_bit.size());
  for (size_t b = 0; b < G->hw_bit.size(); ++b) G->lcol[b] = L.cols[G->hw_bit[b]];
  G->axis_reg_pos.assign(G->K_bits, -1);
  G->axis_lane_pos.assign(G->K_bits, -1);
  G->axis_of_reg.assign(R, -1);
  G->axis_of_lane.assign(5, -1);
  G->cand_bits = 0;
  for (int t = 0; t < G->K_bits; ++t) {
    u64 c = u64(1) << (sh + t);
    for (int b = 0; b < R; ++b) if (G->lcol[b] == c) { G->axis_reg_pos[t] = b; G->axis_of_reg[b] = t; ++G->cand_bits; }
    for (int l = 0; l < 5; ++l) if (G->lcol[R + l] == c) { G->axis_lane_pos[t] = l; G->axis_of_lane[l] = t; }
  }
  // shuffles vs shared memory: the paper observes the shuffle rounds lose once
  // the gathered dimension grows; the planner switches when more than 2
  // candidates per element remain — with 4 candidates the shuffle gather measured 0.3-17%
  // behind the smem one, with 2 even (profiles/r02_sweep_gather_families.jsonl);
  // force_class selects either
  int force = opts ? opts->force_class : -1;
  if (warp_axis && force == LL_CLASS_SHUFFLE)
    fail(LL_ERR_UNSUPPORTED, "gather: L_Wrp^axis != 0 (P:430): the shuffle gather needs the axis off the warps");
  G->smem = warp_axis || force == LL_CLASS_SMEM || (force != LL_CLASS_SHUFFLE && G->cand_bits > 1);
  // smem layout of the staged tile: vector registers, then lanes, then the other
  // registers, then warps (offset order kreg[0,v), klane, kreg[v,R), kwarp), so the
  // staging stores are whole 16-byte vectors with consecutive lanes on consecutive
  // vectors — 4 wavefronts per 512 B, no bank conflicts.  Any linear bijection works
  // for the reads: an output's source is its own logical coordinate with the axis bits
  // replaced, i.e. its own offset with the offset bits holding axis bits (AXPOS)
  // replaced by idx.
  G->smoff.resize(G->lcol.size());
  {
    const int vv = std::min(G->v, R);
    int o = 0;
    for (int b = 0; b < vv; ++b) G->smoff[b] = 1u << o++;
    for (int l = 0; l < 5; ++l) G->smoff[R + l] = 1u << o++;
    for (int b = vv; b < R; ++b) G->smoff[b] = 1u << o++;
    for (size_t b = R + 5; b < G->lcol.size(); ++b) G->smoff[b] = 1u << o++;
  }
  G->axpos.assign(G->K_bits, 0);
  G->axmask = 0;
  for (int t = 0; t < G->K_bits; ++t) {
    int pos = -1;
    for (size_t b = 0; b < G->lcol.size(); ++b)
      if (G->lcol[b] == (u64(1) << (sh + t))) pos = __builtin_ctz(G->smoff[b]);
    if (pos < 0) fail(LL_ERR_UNSUPPORTED, "gather: an in-tile axis bit has no kernel bit (internal)");
    G->axpos[t] = pos;
    G->axmask |= 1u << pos;
  }
  const u64 ne = u64(1) << G->lcol.size();
  const u64 gbytes = G->smem ? ne * u64(w) : 0;
  // TMA staging (cp.async.bulk of the contiguous src and idx tiles, 2 stages) with the
  // line-coalesced σ, on request (opts->pipe = 4 bulk / 5 bulk + bulk store): the default
  // direct loads with 32 bytes per thread beat it on every measured case
  // (profiles/r02_sweep_gather_families.jsonl); force_class = CTA keeps direct loads
  bool contiguous = true;
  {
    int p = 0;
    for (auto& d : L.in) {
      if (dim_level(d.name) <= 2 && p + d.bits > int(G->lcol.size())) contiguous = false;
      p += d.bits;
    }
  }
  G->stages = 2;
  const u64 stage_bytes = ne * u64(w + 4);
  // (round 1 measured the bulk-copy pipeline ahead of direct loads at the layouts' own
  // warp counts from 32 KiB stages, profiles/r01_sweep_gather_tma.jsonl; with extra warps
  // the direct loads win, profiles/r02_sweep_gather_families.jsonl)
  const int pipe = opts ? opts->pipe : 0;
  const bool tma_want = pipe == 4 || pipe == 5;
  G->tma = G->sigma == SIGMA_COALESCED && contiguous && force != LL_CLASS_CTA && tma_want &&
           u64(G->stages) * stage_bytes + gbytes + 16 <= 200 * 1024 && (G->v + ilog2(u64(w))) >= 2;
  G->smem_bytes = int(gbytes + (G->tma ? u64(G->stages) * stage_bytes + 8 * G->stages : 0));
  // outputs through the stage and one cp.async.bulk per tile, as for the scan: for
  // launches of <= 4096 tiles (ramp-bound; measured in profiles/r02_sweep_gather_tma_store.jsonl);
  // LL_GATHER_TMA_STORE=0 / 1 forces either
  {
    const char* e = std::getenv("LL_GATHER_TMA_STORE");
    const bool small = G->grid_bit.size() <= 12;
    G->tma_store = G->tma && (G->w << G->v) >= 4 && (e ? std::string(e) == "1" : (pipe == 5 || small));
  }
  return G;
}

// ---------------------------------------------------------------------------
// Reduce in the fixed fp32 order of reading R-reduce:
// for each in-tile logical axis bit t = 0, 1, ..., K-1 (ascending),
// v <- v(t = 0) + v(t = 1) — a register add, a shfl.bfly or a shared-memory step,
// whichever level of the kernel layout L∘σ holds bit t.  The order is a property of the
// logical tensor alone, so the fp32 bits do not depend on L, on σ or on any plan option.
// ---------------------------------------------------------------------------
std::unique_ptr<ReducePlan> plan_reduce(const Layout& L, int axis, const ll_plan_opts* opts) {
  if (axis < 0 || axis >= int(L.out.size())) fail(LL_ERR_INVALID_ARG, "axis out of range");
  if (!L.distributed()) fail(LL_ERR_UNSUPPORTED, "reduce: L must be a distributed layout (Def 4.10)");
  if (L.in_bits("lane") != 5) fail(LL_ERR_UNSUPPORTED, "reduce: 5 lane bits required");
  if (L.in.size() < 1 || L.in[0].name != "reg") fail(LL_ERR_UNSUPPORTED, "reduce: dims must be reg, lane, warp[, block]");
  auto Rp = std::make_unique<ReducePlan>();
  Rp->L = L; Rp->axis = axis;
  Rp->op = opts ? opts->reduce_op : 0;
  if (Rp->op < 0 || Rp->op > 2) fail(LL_ERR_INVALID_ARG, "reduce_op must be 0 (sum), 1 (max) or 2 (min)");
  const int sh = L.out_shift(axis), ab = L.out[axis].bits;
  const u64 amask = ((u64(1) << ab) - 1) << sh;
  int R = L.in_bits("reg");
  Rp->R = R;
  Rp->Wb = L.in_bits("warp");
  // K: number of in-tile (non-block) axis bits; they must be the low axis bits
  int K = 0;
  for (int k : bits_at_level(L, 0, 2)) if (L.cols[k] & amask) ++K;
  for (int t = 0; t < K; ++t) {
    bool f = false;
    for (int k : bits_at_level(L, 0, 2)) if (L.cols[k] == (u64(1) << (sh + t))) f = true;
    if (!f) fail(LL_ERR_UNSUPPORTED, "reduce: in-tile axis bits must be the low axis bits");
  }
  // kernel layout: faithful (L itself) or line-coalesced σ with non-axis bits
  // preferred in the free lanes (axis bits stay in registers: cheap tree levels)
  int sigma = opts ? opts->sigma : 0;
  Rp->v = std::min(2, R);
  if (sigma == SIGMA_FAITHFUL) {
    Rp->sigma = SIGMA_FAITHFUL;
    for (int k : bits_at_level(L, 0, 2)) Rp->hw_bit.push_back(k);
  } else {
    Rp->sigma = SIGMA_COALESCED;
    Rp->hw_bit = sigma_line(L, Rp->v, [&](int k) { return L.cols[k] != 0 && !(L.cols[k] & amask); });
  }
  // an axis bit on the warps needs a shared-memory step; widen_warps moves only non-axis
  // bits, so this is known before it
  bool warp_axis = false;
  for (size_t b = R + 5; b < Rp->hw_bit.size(); ++b)
    if (L.cols[Rp->hw_bit[b]] & amask) warp_axis = true;
  // default bytes per thread and load path, measured over the Table 4 families x 3 tile
  // shapes x 2 axes at 64 MiB and 1 GiB (profiles/r02_sweep_reduce_scan_families.jsonl):
  // direct LDG loads with 128 bytes per thread (16 warps on a 64 KiB tile, several CTAs per
  // SM) beat the one-CTA-per-SM TMA pipeline on 38 of 48 cases (+4-8% on 64 KiB tiles, up
  // to 2.3x on 8 KiB tiles); the TMA pipeline with 256 bytes per thread stays for 64 KiB
  // tiles whose reduction has a shared-memory (warp) step, where it is even or ahead (up to
  // +21%).  opts->pipe = 4 (bulk) forces the TMA stages, force_class = SHUFFLE the LDG path.
  const bool big_tile = R + 5 + Rp->Wb >= 14;
  const bool tma_auto = warp_axis && big_tile;
  widen_warps(Rp->hw_bit, Rp->R, Rp->Wb, Rp->v, default_int(opts, &ll_plan_opts::thread_bytes, tma_auto ? 256 : 128),
              [&](int k) { return L.cols[k] != 0 && (L.cols[k] & amask) == 0; });
  R = Rp->R;
  // optional smaller CTA tiles (ll_plan_opts.tile_bytes): independent rows to the grid
  const auto rmoved = split_tile(Rp->hw_bit, R, Rp->Wb, 4, opts ? opts->tile_bytes : 0,
                                 [&](int k) { return L.cols[k] != 0 && (L.cols[k] & amask) == 0; });
  const int n = int(Rp->hw_bit.size());
  // classify kernel bits (reduced per level, duplicate) and map each logical axis bit t
  // to the kernel bit that holds it: the steps run in t order
  for (int b = 0; b < n; ++b) {
    u64 c = L.cols[Rp->hw_bit[b]];
    if (c == 0) { Rp->dup_bits.push_back(b); continue; }
    if (!(c & amask)) continue;
    if (b < R) Rp->red_reg.push_back(b);
    else if (b < R + 5) Rp->red_lane.push_back(b - R);
    else Rp->red_warp.push_back(b - R - 5);
  }
  for (int t = 0; t < K; ++t)
    for (int b = 0; b < n; ++b)
      if (L.cols[Rp->hw_bit[b]] == (u64(1) << (sh + t))) Rp->axis_hw.push_back(b);
  if (int(Rp->axis_hw.size()) != K) fail(LL_ERR_UNSUPPORTED, "reduce: axis bit without a kernel bit (internal)");
  auto out_of = [&](u64 c) {
    u64 lower = c & ((u64(1) << sh) - 1);
    u64 a = (c & amask) >> sh;
    u64 upper = c >> (sh + ab);
    return (((upper << (ab - K)) | (a >> K)) << sh) | lower;
  };
  Rp->out_col.assign(n, 0);
  for (int b = 0; b < n; ++b) {
    u64 c = L.cols[Rp->hw_bit[b]];
    bool red = (b < R && std::count(Rp->red_reg.begin(), Rp->red_reg.end(), b)) ||
               (b >= R && b < R + 5 && std::count(Rp->red_lane.begin(), Rp->red_lane.end(), b - R)) ||
               (b >= R + 5 && std::count(Rp->red_warp.begin(), Rp->red_warp.end(), b - R - 5));
    if (c && !red) Rp->out_col[b] = out_of(c);
  }
  for (int k : rmoved) {
    Rp->grid_bit.push_back(k);
    Rp->grid_out.push_back(out_of(L.cols[k]));
  }
  for (int k : bits_at_level(L, 3, 3)) {
    if (L.cols[k] == 0) continue;   // duplicate CTAs are not launched
    Rp->grid_bit.push_back(k);
    Rp->grid_out.push_back(out_of(L.cols[k]));
  }
  Rp->out_elems = u64(1) << (L.d_out() - K);
  // shared memory of the warp steps: the registers still live at the step (not yet
  // reduced, not duplicate) of every thread; shuffles: every live register per lane step
  {
    int dead = 0;
    for (int b : Rp->dup_bits) if (b < R) ++dead;
    Rp->wred_bytes = 0;
    Rp->shfl_per_thread = 0;
    for (int t = 0; t < K; ++t) {
      const int b = Rp->axis_hw[t];
      const int live = R - dead;
      if (b >= R + 5) Rp->wred_bytes = std::max(Rp->wred_bytes, int(u64(4) << (live + 5 + Rp->Wb)));
      else if (b >= R) Rp->shfl_per_thread += 1 << live;
      else ++dead;
    }
  }
  // TMA staging (cp.async.bulk) when the CTA tile is contiguous in HBM (reg, lane, warp
  // are L's lowest packed bits), the stage reads are 16-byte line-coalesced (σ), and two
  // stages fit in smem; force_class = SHUFFLE keeps direct LDG loads
  const u64 tile_bytes = u64(4) << (R + 5 + Rp->Wb);
  bool contiguous = true;
  {
    int p = 0;
    for (auto& d : L.in) {
      if (dim_level(d.name) <= 2 && p + d.bits > R + 5 + Rp->Wb) contiguous = false;
      p += d.bits;
    }
  }
  int force = opts ? opts->force_class : -1;
  const int pipe = opts ? opts->pipe : 0;
  Rp->stages = 0;
  for (int ns = 4; ns >= 2; --ns)
    if (u64(ns) * tile_bytes + u64(Rp->wred_bytes) + 8 * ns <= 200 * 1024) { Rp->stages = ns; break; }
  Rp->tma = Rp->sigma == SIGMA_COALESCED && Rp->v == 2 && contiguous && force != LL_CLASS_SHUFFLE && Rp->stages &&
            (pipe == 4 || pipe == 5 || (pipe == 0 && tma_auto));
  Rp->smem_bytes = Rp->tma ? int(Rp->stages * tile_bytes + Rp->wred_bytes + 8 * Rp->stages) : Rp->wred_bytes;
  return Rp;
}

// ---------------------------------------------------------------------------
// Scan: inclusive prefix sum along `axis` inside each CTA
// tile, fp32, in the order of reading R-scan: for logical axis bit t = 0, 1, ...,
// every element with bit t set adds the value of the last element of the lower half
// of its aligned 2^(t+1)-block.  In the kernel layout L∘σ that partner differs in the
// hardware bit of t (cleared) and the hardware bits of the lower axis bits (set): a
// register read when they are all registers, else a warp shuffle from the partner lane.
// Duplicated (zero-column) positions compute identical values from identical
// inputs and store their own copies.
// ---------------------------------------------------------------------------
std::unique_ptr<ScanPlan> plan_scan(const Layout& L, int axis, const ll_plan_opts* opts) {
  if (axis < 0 || axis >= int(L.out.size())) fail(LL_ERR_INVALID_ARG, "axis out of range");
  if (!L.distributed()) fail(LL_ERR_UNSUPPORTED, "scan: L must be a distributed layout (Def 4.10)");
  if (L.in_bits("lane") != 5) fail(LL_ERR_UNSUPPORTED, "scan: 5 lane bits required");
  if (L.in.size() < 1 || L.in[0].name != "reg") fail(LL_ERR_UNSUPPORTED, "scan: dims must be reg, lane, warp[, block]");
  auto S = std::make_unique<ScanPlan>();
  S->L = L; S->axis = axis;
  S->op = opts ? opts->reduce_op : 0;
  if (S->op < 0 || S->op > 2) fail(LL_ERR_INVALID_ARG, "reduce_op must be 0 (sum), 1 (max) or 2 (min)");
  const int sh = L.out_shift(axis), ab = L.out[axis].bits;
  const u64 amask = ((u64(1) << ab) - 1) << sh;
  int R = L.in_bits("reg");
  S->R = R;
  S->Wb = L.in_bits("warp");
  int K = 0;
  for (int k : bits_at_level(L, 0, 2)) if (L.cols[k] & amask) ++K;
  S->K_bits = K;
  S->v = std::min(2, R);
  const int sigma = opts ? opts->sigma : 0;
  if (sigma == SIGMA_FAITHFUL) {
    S->sigma = SIGMA_FAITHFUL;
    for (int k : bits_at_level(L, 0, 2)) S->hw_bit.push_back(k);
  } else {
    // axis bits stay in registers where possible (register steps need no shuffle)
    S->hw_bit = sigma_line(L, S->v, [&](int k) { return L.cols[k] != 0 && !(L.cols[k] & amask); });
  }
  // default 128 bytes per thread with direct LDG loads: measured over the Table 4 families
  // (profiles/r02_sweep_reduce_scan_families.jsonl) it beats the TMA pipeline (one CTA per
  // SM) on 46 of 48 cases, +5-14% on 64 KiB tiles and up to 1.8x on 8 KiB tiles
  widen_warps(S->hw_bit, S->R, S->Wb, S->v, default_int(opts, &ll_plan_opts::thread_bytes, 128),
              [&](int k) { return L.cols[k] != 0 && (L.cols[k] & amask) == 0; });
  R = S->R;
  // optional smaller CTA tiles (ll_plan_opts.tile_bytes): independent rows to the grid
  const auto smoved = split_tile(S->hw_bit, R, S->Wb, 4, opts ? opts->tile_bytes : 0,
                                 [&](int k) { return L.cols[k] != 0 && (L.cols[k] & amask) == 0; });
  const int n = int(S->hw_bit.size());
  for (int t = 0; t < K; ++t) {
    int b = -1;
    for (int q = 0; q < n; ++q) if (L.cols[S->hw_bit[q]] == (u64(1) << (sh + t))) b = q;
    if (b < 0) fail(LL_ERR_UNSUPPORTED, "scan: in-tile axis bits must be the low axis bits");
    S->axis_hw.push_back(b);
  }
  S->grid_bit = smoved;
  for (int k : bits_at_level(L, 3, 3)) S->grid_bit.push_back(k);
  // shuffles per thread per tile: a step needs them when its bit or a lower axis bit is
  // a lane; one per distinct partner register (slots whose partners coincide share it:
  // the partner has every lower register axis bit set)
  bool lane_below = false, warp_below = false;
  int low_reg_bits = 0;
  for (int t = 0; t < K; ++t) {
    const bool hreg = S->axis_hw[t] < R, hwarp = S->axis_hw[t] >= R + 5;
    if (hwarp || warp_below) S->xs_bytes = (4 << R) * (32 << S->Wb);   // smem step
    else if (!hreg || lane_below) S->shfl_per_thread += 1 << (R - low_reg_bits - (hreg ? 1 : 0));
    if (hwarp) warp_below = true;
    else if (!hreg) lane_below = true;
    else ++low_reg_bits;
  }
  // TMA staging (on request, opts->pipe = 4 / 5) as for the reduce: contiguous CTA tile
  // (reg, lane, warp are L's lowest packed bits), line σ with 16-byte reads, 2-3 stages in
  // smem; force_class = SHUFFLE keeps direct LDG loads
  const u64 tile_bytes = u64(4) << (R + 5 + S->Wb);
  bool contiguous = true;
  {
    int p = 0;
    for (auto& d : L.in) {
      if (dim_level(d.name) <= 2 && p + d.bits > R + 5 + S->Wb) contiguous = false;
      p += d.bits;
    }
  }
  const int force = opts ? opts->force_class : -1;
  const int pipe = opts ? opts->pipe : 0;
  for (int ns = 3; ns >= 2; --ns)
    if (u64(ns) * tile_bytes + u64(S->xs_bytes) + 8 * ns <= 200 * 1024) { S->stages = ns; break; }
  // TMA stages only on request (opts->pipe = 4 bulk / 5 bulk + bulk store)
  S->tma = S->sigma == SIGMA_COALESCED && S->v == 2 && contiguous && force != LL_CLASS_SHUFFLE && S->stages > 0 &&
           (pipe == 4 || pipe == 5);
  // The results can go back into the stage they were read from (each thread rewrites the
  // 16-byte vectors it read) and leave by one cp.async.bulk shared -> global per tile
  // (the dst tile is contiguous like the src tile): the LSU then carries no global
  // stores.  Measured (profiles/r02_sweep_scan.jsonl): +4.5% on the config-4 size (1024
  // tiles, ramp-bound), -4% at 1 GiB (16384 tiles), where the stage held by the in-flight
  // store shortens the load pipeline — so with TMA stages, only for launches of <= 4096
  // tiles, or when opts->pipe = 5 (bulkst) asks for it.  LL_SCAN_TMA_STORE=0 / 1 forces either.
  {
    const char* e = std::getenv("LL_SCAN_TMA_STORE");
    const bool small = S->grid_bit.size() <= 12;
    S->tma_store = S->tma && (e ? std::string(e) == "1" : (pipe == 5 || small));
  }
  S->smem_bytes = S->tma ? int(S->stages * tile_bytes + S->xs_bytes + 8 * S->stages) : S->xs_bytes;
  if (S->smem_bytes > 200 * 1024) fail(LL_ERR_UNSUPPORTED, "scan: tile too large for the shared-memory exchange");
  return S;
}

}  // namespace ll
