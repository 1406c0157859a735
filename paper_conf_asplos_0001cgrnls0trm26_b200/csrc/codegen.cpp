#include <algorithm>
// Specialisation of the sm_100a kernel templates (ll_kernels.cuh): emits the plan
// constants as a `struct P` of compile-time tables and instantiates the entry point.
#include <cstdlib>
#include <sstream>
#include <type_traits>

#include "ll_internal.hpp"

namespace ll {

namespace {

template <class T>
std::string arr(const char* type, const char* name, const std::vector<T>& v) {
  std::ostringstream o;
  o << "  static constexpr " << type << " " << name << "[" << (v.empty() ? 1 : v.size()) << "] = {";
  if (v.empty()) o << "0";
  for (size_t i = 0; i < v.size(); ++i) o << (i ? "," : "") << v[i] << (sizeof(T) == 8 ? "ull" : (std::is_unsigned<T>::value ? "u" : ""));
  o << "};\n";
  return o.str();
}

std::string icon(const char* name, long long v) {
  std::ostringstream o;
  o << "  static constexpr int " << name << " = " << v << ";\n";
  return o.str();
}

int ilog2i(u64 v) { return v ? 63 - __builtin_clzll(v) : -1; }

// Store cache hint for the streaming outputs: 1 = .cs (evict-first; measured +0.5%
// on config 2 and +3% on config 3, profiles/r01_sweep_hints.jsonl), 0 = default
// write-back (env LL_ST_HINT=wb).
int st_hint() {
  const char* e = std::getenv("LL_ST_HINT");
  return (e && std::string(e) == "wb") ? 0 : 1;
}

// grid map: CTA index bit g -> offsets; contiguous when both sides are a run of bits
void emit_grid(std::ostringstream& o, const std::vector<int>& gs, const std::vector<int>& gd, int shift_scale) {
  bool contig = !gs.empty();
  for (size_t g = 0; g < gs.size(); ++g)
    if (gs[g] != gs[0] + int(g) || gd[g] != gd[0] + int(g)) contig = false;
  if (gs.empty()) contig = true;
  o << icon("G", gs.size());
  o << "  static constexpr bool GRID_CONTIG = " << (contig ? "true" : "false") << ";\n";
  o << icon("GRID_LD_SHIFT", gs.empty() ? 0 : gs[0] + shift_scale);
  o << icon("GRID_ST_SHIFT", gd.empty() ? 0 : gd[0] + shift_scale);
  std::vector<u64> ld, st;
  for (size_t g = 0; g < gs.size(); ++g) {
    ld.push_back(u64(1) << (gs[g] + shift_scale));
    st.push_back(u64(1) << (gd[g] + shift_scale));
  }
  o << arr("u64", "GRID_LD", ld) << arr("u64", "GRID_ST", st);
}

}  // namespace

std::string codegen_tile(const ConvPlan& Pl) {
  const TilePlan& T = Pl.tile;
  const int lw = ilog2i(u64(T.w));
  std::ostringstream o;
  o << "// plan: " << describe(Pl).substr(0, 0) << "\nstruct P {\n";
  o << icon("W", T.w) << icon("R", T.R) << icon("WB", T.Wb)
    << icon("NW", std::max<long long>(1, ((1ll << T.R) * T.w) / 4))
    << icon("VLD", T.vld) << icon("VST", T.vst) << icon("XCHG", T.xchg) << icon("THREADS", T.threads());
  o << "  static constexpr bool ISOLATE_SMEM = " << (std::getenv("LL_ISOLATE_SMEM") ? "true" : "false") << ";\n";
  o << icon("ST_HINT", st_hint());
  o << "  static constexpr bool PIPE = " << (T.pipe ? "true" : "false") << ";\n";
  o << "  static constexpr bool STAGED = " << (T.staged ? "true" : "false") << ";\n";
  o << "  static constexpr bool BULK = " << (T.bulk ? "true" : "false") << ";\n";
  o << "  static constexpr bool BCAST = " << (T.bcast ? "true" : "false") << ";\n";
  {
    std::vector<u64> bst;
    for (int u : T.bc_U) bst.push_back(u64(1) << (u + lw));
    const int nk = T.bcast ? int(T.bc_U.size()) - T.bc_v - 5 - T.Wb : 0;
    o << icon("BC_V", T.bc_v) << icon("BC_NK", nk) << arr("u64", "BC_SMW", T.bc_smw) << arr("u64", "BC_SMR", T.bc_smr)
      << arr("u64", "BC_ST", bst);
  }
  o << "  static constexpr bool BULK_ST = " << (T.bulk_st ? "true" : "false") << ";\n";
  o << icon("STAGES", std::max(1, T.bulk_stages)) << icon("TILE_LOG2B", T.n + lw);
  {
    const char* nh = std::getenv("LL_NOHOIST");   // experiment hook: 0 / 1 override
    const bool nohoist = nh ? std::string(nh) == "1" : T.ld_run >= 0;
    o << "  static constexpr bool NOHOIST = " << (nohoist ? "true" : "false") << ";\n";
  }
  o << icon("XBYTES", (long long)(T.smem_elems * u64(T.w)));
  // per-thread-contiguous loads (faithful σ) re-use sectors across instructions
  o << "  static constexpr bool LD_L1 = " << (T.sigma == SIGMA_FAITHFUL ? "true" : "false") << ";\n";
  // XOR-copy plans: a src column may reach below the vector (bits [0, VLD)): that part is
  // an element XOR inside the aligned src vector (in-vector XOR, LD_LO / GRID_LD_LO),
  // the rest a byte offset
  const u64 lowm = (u64(1) << T.vld) - 1;
  bool invec = false;
  for (size_t b = size_t(T.vld); b < T.ld_xcol.size(); ++b) invec |= (T.ld_xcol[b] & lowm) != 0;
  for (u64 c : T.grid_src_xcol) invec |= (c & lowm) != 0;
  std::vector<u64> ldc, stc;
  std::vector<uint32_t> ldlo, gridlo;
  for (int b = 0; b < T.n; ++b) {
    const bool vecbit = b < T.vld;
    ldc.push_back(T.ld_xcol.empty() ? (u64(1) << (T.ld_bit[b] + lw))
                                    : ((vecbit ? T.ld_xcol[b] : (T.ld_xcol[b] & ~lowm)) << lw));
    ldlo.push_back(T.ld_xcol.empty() || vecbit ? 0u : uint32_t(T.ld_xcol[b] & lowm));
    stc.push_back(u64(1) << (T.st_bit[b] + lw));
  }
  for (u64 c : T.grid_src_xcol) gridlo.push_back(uint32_t(c & lowm));
  o << arr("u64", "LD_COL", ldc) << arr("u64", "ST_COL", stc);
  o << "  static constexpr bool LD_XOR = " << (T.ld_xcol.empty() ? "false" : "true") << ";\n";
  o << "  static constexpr bool LD_INVEC = " << (invec ? "true" : "false") << ";\n";
  o << arr("u32", "LD_LO", ldlo) << arr("u32", "GRID_LD_LO", gridlo);
  if (T.grid_src_xcol.empty()) {
    emit_grid(o, T.grid_src_bit, T.grid_dst_bit, lw);
  } else {
    // XOR grid: per-bit src / dst offsets (never contiguous shifts)
    std::vector<u64> ld, st;
    for (size_t g = 0; g < T.grid_dst_bit.size(); ++g) {
      ld.push_back((T.grid_src_xcol[g] & ~lowm) << lw);
      st.push_back(u64(1) << (T.grid_dst_bit[g] + lw));
    }
    o << icon("G", T.grid_dst_bit.size()) << "  static constexpr bool GRID_CONTIG = false;\n"
      << icon("GRID_LD_SHIFT", 0) << icon("GRID_ST_SHIFT", 0) << arr("u64", "GRID_LD", ld) << arr("u64", "GRID_ST", st);
  }
  // broadcast destinations: every value is stored at 2^|rep| replica offsets (bytes).
  // The lowest rep_lo (<= 4) replica bits are unrolled (stores to neighbouring offsets
  // per vector); the remaining ones are CTA-index bits above the data tiles' (REP_HI:
  // one offset per bit, XOR-combined by the replica group), so any number of zero
  // columns stays on the specialised kernel with enough CTAs to fill the GPU.
  std::vector<int> rb = T.rep_bits;
  std::sort(rb.begin(), rb.end());
  const size_t nlo = std::min<size_t>(size_t(T.rep_lo), rb.size());
  std::vector<u64> rep(size_t(1) << nlo, 0), rep_hi;
  for (size_t r = 0; r < rep.size(); ++r)
    for (size_t t = 0; t < nlo; ++t)
      if ((r >> t) & 1) rep[r] |= u64(1) << (rb[t] + lw);
  for (size_t t = nlo; t < rb.size(); ++t) rep_hi.push_back(u64(1) << (rb[t] + lw));
  o << icon("NREP", rep.size()) << arr("u64", "REP_OFF", rep)
    << icon("NREP_HI_BITS", rep_hi.size()) << arr("u64", "REP_HI", rep_hi);
  // element permutations around a sub-word shuffle (plan_shuffle_eperm)
  o << "  static constexpr bool EPERM = " << (T.pre_eperm.empty() ? "false" : "true") << ";\n"
    << arr("int", "PRE_EPERM", T.pre_eperm) << arr("int", "POST_EPERM", T.post_eperm);
  // REGPERM
  o << arr("int", "PERM", T.perm);
  // SHUFFLE
  o << icon("NSLOT", T.nslot) << icon("UW", std::max(1, T.unit_elems * T.w / 4)) << icon("ROUNDS", T.rounds)
    << icon("NPRE", T.pre_x.size()) << icon("NPOST", T.post_x.size());
  o << arr("int", "SEND_SLOT", T.send_slot) << arr("int", "RECV_SLOT", T.recv_slot)
    << arr("u32", "SRC_LANE0", T.src_lane0)
    << arr("u32", "SRC_LANE_COL", std::vector<uint32_t>(T.src_lane_col, T.src_lane_col + 5))
    << arr("u32", "PRE_LMASK", T.pre_lmask) << arr("int", "PRE_X", T.pre_x)
    << arr("u32", "POST_LMASK", T.post_lmask) << arr("int", "POST_X", T.post_x);
  // SMEM
  o << icon("SV", T.sm_v) << arr("int", "VSLOT_LD", T.vec_slot_ld) << arr("int", "VSLOT_ST", T.vec_slot_st)
    << arr("u64", "SMOFF_LD", T.smoff_ld) << arr("u64", "SMOFF_ST", T.smoff_st);
  // stmatrix / ldmatrix sides (Thm 5.1)
  o << icon("SMI_LD", T.smi_ld) << icon("SMI_ST", T.smi_st)
    << icon("NMW", T.w <= 4 ? ilog2i(u64(4 / T.w)) : 0)
    << arr("int", "MWORD_LD", T.mat_word_ld) << arr("int", "MWORD_ST", T.mat_word_st)
    << icon("NMSEL_LD", T.mat_sel_ld.size()) << icon("NMSEL_ST", T.mat_sel_st.size())
    << arr("int", "MSEL_LD", T.mat_sel_ld) << arr("int", "MSEL_ST", T.mat_sel_st);
  o << "};\n";
  if (Pl.peer_shift >= 0) {
    // DEVICE plan executed as peer stores (N4): global dst offsets, window per rank
    const int sh = Pl.peer_shift + lw;
    o << "extern \"C\" __global__ void __launch_bounds__(" << T.threads()
      << ") ll_tile_peer_kernel(const u8* __restrict__ src, const __grid_constant__ LLPeers peers, u64 ntiles,"
         " u64 tile0) {\n"
      << "  ll_tile_body<P, DstPeers<" << sh << ">, " << (Pl.peer_reg ? "true" : "false") << ">(src, DstPeers<" << sh
      << ">(&peers), ntiles, tile0);\n}\n";
  } else {
    o << "extern \"C\" __global__ void __launch_bounds__(" << T.threads();
    if (T.min_blocks > 0) o << ", " << T.min_blocks;   // ptxas register cap (plan_exchange)
    o << ") ll_tile_kernel(const u8* __restrict__ src, u8* __restrict__ dst, u64 ntiles) {\n"
      << "  ll_tile_body<P>(src, DstLocal(dst), ntiles);\n}\n";
  }
  return o.str();
}

// Minimum-blocks hint for the gather / scan / reduce kernels: `dflt` CTAs per SM
// (0 = none); LL_AUX_MIN_BLOCKS=k overrides it (0 = none) for experiments.
static std::string aux_min_blocks(int dflt = 0) {
  const char* e = std::getenv("LL_AUX_MIN_BLOCKS");
  const int k = e ? std::atoi(e) : dflt;
  return k > 0 ? ", " + std::to_string(k) : std::string();
}

std::string codegen_gather(const GatherPlan& G) {
  std::ostringstream o;
  const int n = int(G.hw_bit.size());
  o << "struct P {\n";
  o << icon("W", G.w) << icon("R", G.R) << icon("WB", G.Wb)
    << icon("NW", std::max<long long>(1, ((1ll << G.R) * G.w) / 4)) << icon("VLD", G.v);
  o << "  static constexpr bool LD_L1 = " << (G.sigma == SIGMA_FAITHFUL ? "true" : "false") << ";\n";
  o << icon("ST_HINT", st_hint());
  std::vector<u64> ldc;
  for (int b = 0; b < n; ++b) ldc.push_back(u64(1) << G.hw_bit[b]);   // element offsets
  o << arr("u64", "LD_COL", ldc);
  emit_grid(o, G.grid_bit, G.grid_bit, 0);
  o << icon("KBITS", G.K_bits) << icon("CBITS", G.cand_bits);
  o << arr("int", "AXIS_OF_LANE", G.axis_of_lane) << arr("int", "AXIS_LANE_POS", G.axis_lane_pos);
  // candidate bits: the register bits that carry axis bits, in ascending order
  std::vector<int> cand_reg, axis_cand_pos(G.K_bits, -1), axis_of_reg = G.axis_of_reg;
  for (int b = 0; b < G.R; ++b)
    if (G.axis_of_reg[b] >= 0) { axis_cand_pos[G.axis_of_reg[b]] = int(cand_reg.size()); cand_reg.push_back(b); }
  o << arr("int", "AXIS_CAND_POS", axis_cand_pos) << arr("int", "CAND_REG", cand_reg)
    << arr("int", "AXIS_OF_REG", axis_of_reg);
  o << "  template <int E> static constexpr u32 axis_of_slot() { u32 a = 0;"
       " for (int b = 0; b < R; ++b) if (((E >> b) & 1) && AXIS_OF_REG[b] >= 0) a ^= 1u << AXIS_OF_REG[b]; return a; }\n";
  o << "  template <int E> static constexpr u32 cand_of_slot() { u32 c = 0;"
       " for (int i = 0; i < CBITS; ++i) if ((E >> CAND_REG[i]) & 1) c |= 1u << i; return c; }\n";
  o << "  static constexpr bool GATHER_SMEM = " << (G.smem ? "true" : "false") << ";\n";
  o << "  static constexpr bool TMA = " << (G.tma ? "true" : "false") << ";\n";
  o << "  static constexpr bool TMA_STORE = " << (G.tma_store ? "true" : "false") << ";\n";
  o << "  static constexpr unsigned STAGES = " << std::max(1, G.stages) << "u;\n";
  // staging stores as 2^v-element vectors when the thread's vector registers are
  // consecutive in the logical tile order (line σ: the lowest logical bits)
  int smv = 0;
  while (smv < G.v && smv < int(G.smoff.size()) && G.smoff[smv] == (1u << smv)) ++smv;
  o << icon("SMV", smv);
  o << arr("u32", "SMOFF", G.smoff) << "  static constexpr u32 AXMASK = " << G.axmask << "u;\n"
    << arr("int", "AXPOS", G.axpos);
  o << "  template <int E> static constexpr u32 smoff_of_slot() { u32 s = 0;"
       " for (int b = 0; b < R; ++b) if ((E >> b) & 1) s ^= SMOFF[b]; return s; }\n";
  o << "  template <int E, int C> static constexpr int slot_of() { int s = E;"
       " for (int i = 0; i < CBITS; ++i) { s &= ~(1 << CAND_REG[i]); if ((C >> i) & 1) s |= 1 << CAND_REG[i]; } return s; }\n";
  o << "};\n";
  o << "extern \"C\" __global__ void __launch_bounds__(" << (32 << G.Wb) << aux_min_blocks()
    << ") ll_gather_kernel(const u8* __restrict__ src, const u8* __restrict__ idx, u8* __restrict__ dst, u64 ntiles) {\n"
    << "  ll_gather_body<P>(src, idx, dst, ntiles);\n}\n";
  return o.str();
}

std::string codegen_scan(const ScanPlan& S) {
  std::ostringstream o;
  o << "struct P {\n";
  o << icon("W", 4) << icon("R", S.R) << icon("WB", S.Wb) << icon("VLD", S.v) << icon("NW", 1 << S.R)
    << icon("OP", S.op);
  o << "  static constexpr bool LD_L1 = " << (S.sigma == SIGMA_FAITHFUL ? "true" : "false") << ";\n";
  o << icon("ST_HINT", st_hint());
  std::vector<u64> ldc;
  for (int b : S.hw_bit) ldc.push_back(u64(4) << b);
  o << arr("u64", "LD_COL", ldc);
  emit_grid(o, S.grid_bit, S.grid_bit, 2);
  o << icon("KB", S.K_bits) << arr("int", "AXIS_HW", S.axis_hw);
  o << "  static constexpr bool TMA = " << (S.tma ? "true" : "false") << ";\n";
  o << "  static constexpr bool TMA_STORE = " << (S.tma_store ? "true" : "false") << ";\n";
  o << "  static constexpr unsigned STAGES = " << std::max(1, S.stages) << "u;\n";
  o << "  static constexpr unsigned XS_BYTES = " << S.xs_bytes << "u;\n";
  o << "};\n";
  // scans without a shared-memory warp step (axis bits on registers and lanes) ask for
  // 2 CTAs per SM: +0.3-3.5% on all 24 such Table 4 cases (families x tiles x 64 MiB /
  // 1 GiB), mixed with a warp step (profiles/r02_sweep_families_aux_min_blocks.jsonl)
  o << "extern \"C\" __global__ void __launch_bounds__(" << (32 << S.Wb) << aux_min_blocks(S.xs_bytes == 0 ? 2 : 0)
    << ") ll_scan_kernel(const u8* __restrict__ src, u8* __restrict__ dst, u64 ntiles) {\n"
    << "  ll_scan_body<P>(src, dst, ntiles);\n}\n";
  return o.str();
}

std::string codegen_reduce(const ReducePlan& Rp) {
  std::ostringstream o;
  o << "struct P {\n";
  const int R = Rp.R, n = int(Rp.hw_bit.size());
  o << icon("W", 4) << icon("R", R) << icon("WB", Rp.Wb) << icon("VLD", Rp.v) << icon("OP", Rp.op);
  o << "  static constexpr bool LD_L1 = " << (Rp.sigma == SIGMA_FAITHFUL ? "true" : "false") << ";\n";
  o << "  static constexpr bool TMA = " << (Rp.tma ? "true" : "false") << ";\n";
  o << "  static constexpr unsigned WRED_BYTES = " << Rp.wred_bytes << "u;\n";
  o << "  static constexpr unsigned STAGES = " << std::max(1, Rp.stages) << "u;\n";
  std::vector<u64> ldc;
  for (int b = 0; b < n; ++b) ldc.push_back(u64(4) << Rp.hw_bit[b]);
  o << arr("u64", "LD_COL", ldc);
  emit_grid(o, Rp.grid_bit, Rp.grid_bit, 2);
  o << arr("u64", "GRID_OUT", Rp.grid_out) << arr("u64", "OUT_COL", Rp.out_col);
  int regmask = 0, dupreg = 0;
  uint32_t nolane = 0, nowarp = 0;
  for (int b : Rp.red_reg) regmask |= 1 << b;
  for (int b : Rp.red_lane) nolane |= 1u << b;
  for (int b : Rp.red_warp) nowarp |= 1u << b;
  for (int k : Rp.dup_bits) {
    if (k < R) dupreg |= 1 << k;
    else if (k < R + 5) nolane |= 1u << (k - R);
    else nowarp |= 1u << (k - R - 5);
  }
  o << icon("RED_REG_MASK", regmask) << icon("DUP_REG_MASK", dupreg)
    << icon("KB", Rp.axis_hw.size()) << arr("int", "AXIS_HW", Rp.axis_hw);
  o << "  static constexpr u32 NOSTORE_LANE_MASK = " << nolane << "u;\n"
    << "  static constexpr u32 NOSTORE_WARP_MASK = " << nowarp << "u;\n";
  o << "  template <int E> static constexpr u64 out_of_slot() { u64 c = 0; for (int b = 0; b < R; ++b) if ((E >> b) & 1) c ^= OUT_COL[b]; return c; }\n";
  o << "};\n";
  o << "extern \"C\" __global__ void __launch_bounds__(" << (32 << Rp.Wb) << aux_min_blocks()
    << ") ll_reduce_kernel(const float* __restrict__ src, float* __restrict__ dst, u64 ntiles) {\n"
    << "  ll_reduce_body<P>(src, dst, ntiles);\n}\n";
  return o.str();
}

}  // namespace ll
