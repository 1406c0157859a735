// Host emulation of a specialised tile plan's schedule (test hook ll_plan_simulate).
// It executes exactly the tables the kernel is specialised with — σ_ld / σ_st
// addresses, the pre / post conditional-swap networks, the shuffle rounds with their
// source lanes and slots, the swizzled smem offsets — one warp at a time, so the
// planner can be validated without a GPU.  It is never used by ll_convert.
#include <cstring>

#include "ll_internal.hpp"

namespace ll {

namespace {
struct struct_off { u64 thr, reg, elem; };
}  // namespace

void simulate_tile(const ConvPlan& P, const uint8_t* src, uint8_t* dst) {
  if (P.exec != EXEC_TILE) fail(LL_ERR_UNSUPPORTED, "simulate: not a tile plan");
  const TilePlan& T = P.tile;
  const int w = T.w, R = T.R, n = T.n;
  const int E = 1 << R, NT = T.threads();
  const u64 ntiles = u64(1) << T.grid_dst_bit.size();
  // Address arithmetic exactly as ll_tile_body forms it: thread part (lane / warp
  // columns) XOR the tile base; the register part of vector K (bits >= vld) added —
  // or XORed for XOR-copy plans (LD_XOR) — and element i of the vector at +i.
  const bool ld_xor = !T.ld_xcol.empty();
  auto ld_col = [&](int b) { return ld_xor ? T.ld_xcol[b] : (u64(1) << T.ld_bit[b]); };
  auto ld_off = [&](u64 hw) {
    const u64 vmask = (u64(1) << T.vld) - 1;
    u64 thr = 0, reg = 0;
    for (int b = R; b < n; ++b) if ((hw >> b) & 1) thr ^= ld_col(b);
    for (int b = T.vld; b < R; ++b) if ((hw >> b) & 1) reg ^= ld_col(b);
    return struct_off{thr, reg, hw & vmask};
  };
  std::vector<uint64_t> in(size_t(NT) * E), out(size_t(NT) * E);
  std::vector<uint8_t> smem(T.xchg == X_SMEM ? T.smem_elems * w : 0);
  auto getv = [&](const uint8_t* p) { uint64_t v = 0; std::memcpy(&v, p, w); return v; };
  for (u64 t = 0; t < ntiles; ++t) {
    u64 sb = 0, db = 0;
    for (size_t g = 0; g < T.grid_dst_bit.size(); ++g)
      if ((t >> g) & 1) {
        sb ^= T.grid_src_xcol.empty() ? (u64(1) << T.grid_src_bit[g]) : T.grid_src_xcol[g];
        db |= u64(1) << T.grid_dst_bit[g];
      }
    for (int th = 0; th < NT; ++th)
      for (int e = 0; e < E; ++e) {
        u64 hw = u64(e) | (u64(th) << R);
        struct_off a = ld_off(hw);
        u64 base = sb ^ a.thr;
        // XOR-copy plans: as the kernel does it — an aligned vector load at the high part
        // of the XOR, element e taken from position e ^ (low part) (in-vector XOR, when a
        // swizzle reaches below the vector)
        const u64 vmask = (u64(1) << T.vld) - 1;
        const u64 x = base ^ a.reg;
        u64 idx = ld_xor ? ((x & ~vmask) + (a.elem ^ (x & vmask))) : (base + a.reg + a.elem);
        in[size_t(th) * E + e] = getv(src + idx * w);
      }
    if (T.bcast) {
      // broadcast stores in dst order: data to smem in dst-data order, then read along
      // the store tile U (vector, lanes, warps, per-thread vectors) and stored at every
      // remaining replica offset
      std::vector<uint8_t> sm((u64(1) << n) * w);
      for (int th = 0; th < NT; ++th)
        for (int e = 0; e < E; ++e) {
          u64 hw = u64(e) | (u64(th) << R);
          u64 so = 0;
          for (int b = 0; b < n; ++b) if ((hw >> b) & 1) so ^= T.bc_smw[b];
          std::memcpy(&sm[so * w], &in[size_t(th) * E + e], w);
        }
      const int nU = int(T.bc_U.size());
      for (u64 pos = 0; pos < (u64(1) << nU); ++pos) {
        u64 so = 0, d = db;
        for (int u = 0; u < nU; ++u)
          if ((pos >> u) & 1) { so ^= T.bc_smr[u]; d ^= u64(1) << T.bc_U[u]; }
        for (u64 rp = 0; rp < (u64(1) << T.rep_bits.size()); ++rp) {
          u64 ro = 0;
          for (size_t q = 0; q < T.rep_bits.size(); ++q) if ((rp >> q) & 1) ro |= u64(1) << T.rep_bits[q];
          std::memcpy(dst + (d ^ ro) * w, &sm[so * w], w);
        }
      }
      continue;
    }
    if (T.xchg == X_COPY) {
      out = in;
    } else if (T.xchg == X_REGPERM) {
      for (int th = 0; th < NT; ++th)
        for (int e = 0; e < E; ++e) out[size_t(th) * E + e] = in[size_t(th) * E + T.perm[e]];
    } else if (T.xchg == X_SHUFFLE) {
      const int U = T.unit_elems;
      if (!T.pre_eperm.empty()) {
        std::vector<uint64_t> tmp(in.size());
        for (int th = 0; th < NT; ++th)
          for (int e = 0; e < E; ++e) tmp[size_t(th) * E + e] = in[size_t(th) * E + T.pre_eperm[e]];
        in.swap(tmp);
      }
      for (int wp = 0; wp < (1 << T.Wb); ++wp) {
        // pre network: slot j <-> j ^ X when parity(lane & mask)
        auto net = [&](std::vector<uint64_t>& buf, const std::vector<uint32_t>& mk, const std::vector<int>& xs) {
          for (size_t s = 0; s < xs.size(); ++s)
            for (int l = 0; l < 32; ++l) {
              if (!parity(u64(l) & mk[s])) continue;
              uint64_t* r = &buf[size_t(wp * 32 + l) * E];
              for (int j = 0; j < T.nslot; ++j) {
                int k = j ^ xs[s];
                if (k > j) for (int q = 0; q < U; ++q) std::swap(r[j * U + q], r[k * U + q]);
              }
            }
        };
        net(in, T.pre_lmask, T.pre_x);
        for (int rr = 0; rr < T.rounds; ++rr) {
          int S = T.send_slot[rr];
          uint64_t sent[32][8];
          for (int l = 0; l < 32; ++l)
            for (int q = 0; q < U; ++q) sent[l][q] = in[size_t(wp * 32 + l) * E + S * U + q];
          for (int l = 0; l < 32; ++l) {
            uint32_t lx = 0;
            for (int b = 0; b < 5; ++b) if ((l >> b) & 1) lx ^= T.src_lane_col[b];
            int sl = int((T.src_lane0[rr] ^ lx) & 31);
            for (int q = 0; q < U; ++q) in[size_t(wp * 32 + l) * E + S * U + q] = sent[sl][q];
          }
        }
        for (int l = 0; l < 32; ++l)
          for (int rr = 0; rr < T.rounds; ++rr)
            for (int q = 0; q < U; ++q)
              out[size_t(wp * 32 + l) * E + T.recv_slot[rr] * U + q] = in[size_t(wp * 32 + l) * E + T.send_slot[rr] * U + q];
        net(out, T.post_lmask, T.post_x);
      }
      if (!T.post_eperm.empty()) {
        std::vector<uint64_t> tmp(out.size());
        for (int th = 0; th < NT; ++th)
          for (int e = 0; e < E; ++e) tmp[size_t(th) * E + e] = out[size_t(th) * E + T.post_eperm[e]];
        out.swap(tmp);
      }
    } else {
      for (int th = 0; th < NT; ++th)
        for (int e = 0; e < E; ++e) {
          u64 hw = u64(e) | (u64(th) << R);
          u64 so = 0;
          for (int b = 0; b < n; ++b) if ((hw >> b) & 1) so ^= T.smoff_ld[b];
          std::memcpy(&smem[so * w], &in[size_t(th) * E + e], w);
        }
      for (int th = 0; th < NT; ++th)
        for (int e = 0; e < E; ++e) {
          u64 hw = u64(e) | (u64(th) << R);
          u64 so = 0;
          for (int b = 0; b < n; ++b) if ((hw >> b) & 1) so ^= T.smoff_st[b];
          uint64_t v = 0;
          std::memcpy(&v, &smem[so * w], w);
          out[size_t(th) * E + e] = v;
        }
    }
    for (u64 rp = 0; rp < (u64(1) << T.rep_bits.size()); ++rp) {
      u64 ro = 0;
      for (size_t t = 0; t < T.rep_bits.size(); ++t) if ((rp >> t) & 1) ro |= u64(1) << T.rep_bits[t];
      for (int th = 0; th < NT; ++th)
        for (int e = 0; e < E; ++e) {
          u64 hw = u64(e) | (u64(th) << R);
          const u64 vmask = (u64(1) << T.vst) - 1;
          u64 thr = 0, reg = 0;
          for (int b = R; b < n; ++b) if ((hw >> b) & 1) thr ^= u64(1) << T.st_bit[b];
          for (int b = T.vst; b < R; ++b) if ((hw >> b) & 1) reg ^= u64(1) << T.st_bit[b];
          u64 idx = (db ^ thr) + (reg ^ ro) + (hw & vmask);
          std::memcpy(dst + idx * w, &out[size_t(th) * E + e], w);
        }
    }
  }
}

}  // namespace ll
