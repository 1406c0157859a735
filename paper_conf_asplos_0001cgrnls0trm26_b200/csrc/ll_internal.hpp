// Internal declarations of the linear-layout library (host side).
//
// Layer map:
//   f2      — F2 vector/matrix helpers over uint64 columns (§2.4)
//   Layout  — labelled linear layouts (Def 4.1) and their algebra
//             (Defs 4.2-4.5)
//   plan    — conversion planner: pull map Q = A^+ ∘ B, class selection
//             (P:350-373), kernel decomposition, shuffle plan and
//             optimal swizzle; gather and
//             reduce plans
//   codegen — specialisation of the sm_100a kernel templates (ll_kernels.cuh)
//   jit     — NVRTC compilation + cubin cache + cudaLibrary loading
//   capi    — the C ABI of include/ll.h
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <map>
#include <memory>
#include <mutex>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/ll.h"

namespace ll {

using u64 = uint64_t;

// Error carrying an ll_status across internal layers; never crosses the ABI.
struct Error : std::runtime_error {
  ll_status st;
  Error(ll_status s, const std::string& m) : std::runtime_error(m), st(s) {}
};
[[noreturn]] void fail(ll_status s, const std::string& msg);
void set_last_error(const std::string& msg);

inline int popc(u64 v) { return __builtin_popcountll(v); }
inline int lead(u64 v) { return 63 - __builtin_clzll(v); }
inline bool parity(u64 v) { return popc(v) & 1; }

// ------------------------------------------------------------------ F2 helpers
// Row-echelon basis keyed by leading bit, tracking for every stored vector the
// combination (over some index space) that produced it.
struct Echelon {
  u64 vec[64] = {0};
  u64 comb[64] = {0};
  bool has[64] = {false};
  int rank = 0;
  // Reduce v (with running combination c); returns the residue.
  u64 reduce(u64 v, u64* c = nullptr) const {
    while (v) {
      int l = lead(v);
      if (!has[l]) return v;
      v ^= vec[l];
      if (c) *c ^= comb[l];
    }
    return 0;
  }
  // Insert v (with combination c); returns true if it was independent.
  bool insert(u64 v, u64 c = 0) {
    v = reduce(v, &c);
    if (!v) return false;
    int l = lead(v);
    has[l] = true; vec[l] = v; comb[l] = c; ++rank;
    return true;
  }
  bool contains(u64 v) const { return reduce(v) == 0; }
};

// ------------------------------------------------------------------ layouts
struct Dim {
  std::string name;
  int bits;
  bool operator==(const Dim& o) const { return name == o.name && bits == o.bits; }
  bool operator!=(const Dim& o) const { return !(*this == o); }
};

// Hardware level of an input dim (reg < lane < warp < block < dev).  "offset"
// (memory layouts, Def 4.14) lives at the block level.  Unknown names: -1.
int dim_level(const std::string& name);

struct Layout {
  std::vector<Dim> in, out;
  // cols[k]: logical flat index (row-major over `out`, last dim fastest)
  // hit by hardware bit k (hardware flat order: first input dim lowest).
  std::vector<u64> cols;

  int d_in() const;
  int d_out() const;
  int in_pos(const std::string& name) const;   // first hardware bit of dim, -1
  int in_bits(const std::string& name) const;  // 0 if absent
  int out_shift(int out_index) const;          // flat shift of output dim
  u64 apply(u64 h) const {
    u64 x = 0;
    for (size_t k = 0; k < cols.size(); ++k)
      if ((h >> k) & 1) x ^= cols[k];
    return x;
  }
  int rank() const;
  bool surjective() const { return rank() == d_out(); }
  bool injective() const { return rank() == d_in(); }
  bool distributed() const;   // Def 4.10
  bool memory() const;        // Def 4.14
  bool unit_columns() const;  // every column a single bit (a bijective permutation)
};

// Slack-zero right inverse: per logical flat bit t, the hardware
// index of the solution with free variables 0 and pivots in ascending column order.
std::vector<u64> right_inverse_cols(const Layout& L);
u64 apply_cols(const std::vector<u64>& cols, u64 v);
// Basis of ker(L) (hardware vectors).
std::vector<u64> kernel_basis(const Layout& L);

Layout compose(const Layout& outer, const Layout& inner);     // Def 4.2
Layout invert(const Layout& L);                                // Def 4.5
Layout product(const Layout& L1, const Layout& L2);            // Def 4.3
Layout left_divide(const Layout& M, const Layout& M1);         // Def 4.4
Layout make_blocked(const std::vector<int>& shape, const std::vector<int>& spt, const std::vector<int>& tpw,
                    const std::vector<int>& wpc, const std::vector<int>& order);   // Prop 9.1
Layout make_mma_acc(int M, int N, int warps_m, int warps_n);                     // Prop 9.2
Layout make_mma_swizzle(int m, int n, int vec, int per_phase, int max_phase);    // Def 4.11
Layout make_slice(const Layout& L, int dim);                                     // Prop 4.8
Layout make_mma_operand(int is_rhs, int rows, int cols, int bitwidth, int warps_m, int warps_n);  // Prop 9.2
Layout make_tmem_32x32b(int M, int N);                                           // tcgen05.ld
Layout make_tmem(const std::string& shape, int M, int N);                        // tcgen05.ld families

// ------------------------------------------------------------------ plans
enum ExecKind { EXEC_NOOP = 0, EXEC_TILE = 1, EXEC_GENERIC = 2, EXEC_DEVICE = 3 };
enum TileXchg { X_COPY = 0, X_REGPERM = 1, X_SHUFFLE = 2, X_SMEM = 3 };
enum SigmaMode { SIGMA_COALESCED = 0, SIGMA_FAITHFUL = 1 };
enum SmemInstr { SMI_VEC = 0, SMI_MAT = 1, SMI_MATT = 2 };

// Kernel decomposition of a conversion whose pull map is a bit permutation:
// a CTA owns `n` tile bits; kernel hardware inside the CTA is (R reg bits,
// 5 lane bits, Wb warp bits).  For every kernel hardware bit b:
//   ld_bit[b] = src packed bit it loads from (L_ld = A ∘ σ_ld), lcol_ld[b] = A.col
//   st_bit[b] = dst packed bit it stores to  (L_st = B ∘ σ_st), lcol_st[b] = B.col
// Kernel bit order: reg 0..R-1, lane 0..4, warp 0..Wb-1.
struct TilePlan {
  int w = 4;            // element bytes
  int n = 0;            // tile bits
  int R = 0, Wb = 0;    // kernel reg / warp bits (lanes = 5)
  int vld = 0, vst = 0; // elements per global vector = 1 << v
  std::vector<int> ld_bit, st_bit;
  std::vector<u64> lcol_ld, lcol_st;
  std::vector<int> grid_src_bit, grid_dst_bit;   // CTA index bit g -> packed bits
  std::vector<int> rep_bits;   // dst packed bits with zero columns in B: store replicas
  int rep_lo = 0;              // replica bits unrolled per store; the rest are grid bits
  // Linear (XOR) copy plans: the src index of kernel bit b / grid bit g is an arbitrary
  // F2 combination Q(dst bit) (swizzled memory layouts, Def 4.14; broadcast).  When
  // non-empty these replace 1 << ld_bit / 1 << grid_src_bit.
  std::vector<u64> ld_xcol, grid_src_xcol;
  int ld_run = -1;      // linear tiles: low src bits loaded as contiguous runs (c)
  int st_run = -1;      // linear tiles: low dst bits stored as contiguous runs (cs)
  int sigma = SIGMA_COALESCED;
  int xchg = X_COPY;
  bool pipe = false;    // X_SMEM: next tile's loads issued before this tile's stores
  int min_blocks = 0;   // __launch_bounds__ minimum resident CTAs per SM (0 = none)
  bool staged = false;  // X_SMEM: src tiles streamed by cp.async into two raw smem stages
  bool bulk = false;    // X_SMEM: src tiles (contiguous) streamed by cp.async.bulk into raw stages
  bool bulk_st = false; // ... and dst tiles (contiguous) leave by cp.async.bulk from a dst stage
  int bulk_stages = 0;
  // Broadcast stores in dst order (bcast): when B has zero columns among its lowest
  // v + 5 dst bits (inside the 16-byte store vector or the lanes), the data tile goes
  // through shared memory in dst-data order and is read back in full dst order — the
  // replica (zero-column) bits address the same smem element — so every thread stores
  // whole 16-byte vectors and every warp 512 contiguous bytes.  bc_U = the store tile's
  // dst bits (data bits of the tile ∪ low replica bits, ascending: vector, lanes, warps,
  // then per-thread vectors); bc_smr[u] = smem element offset of U bit u (0 for a
  // replica bit); bc_smw[b] = smem element offset written by kernel load bit b.
  bool bcast = false;
  int bc_v = 0;
  std::vector<int> bc_U;
  std::vector<u64> bc_smr, bc_smw;

  // --- REGPERM: out slot e <- in slot perm[e]
  std::vector<int> perm;

  // --- SHUFFLE; units of `unit_elems` elements (one 32-bit word for
  // w<4, one element for w>=4); all unit indices are register-unit indices.
  int unit_elems = 1, nslot = 0;
  std::vector<u64> V, I, E, F, G, Rb;          // logical vectors (describe)
  int rounds = 0;
  std::vector<int> send_slot, recv_slot;       // per round (after pre-permutation)
  std::vector<uint32_t> src_lane0;             // per round: source lane for lane 0
  uint32_t src_lane_col[5] = {0, 0, 0, 0, 0};  // linear part: lane bit t -> XOR
  std::vector<uint32_t> pre_lmask, post_lmask; // per stage: lane mask (parity predicate)
  std::vector<int> pre_x, post_x;              // per stage: slot XOR constant
  // Sub-word elements (w < 4) whose common 32-bit unit V is not the lowest register
  // bits of a side: thread-local element permutations (byte permutes) around the
  // shuffle.  pre_eperm[e'] = the loaded register element that becomes element e' of
  // the shuffle's input; post_eperm[e] = the shuffle-output element stored as e.
  // Empty = identity.
  std::vector<int> pre_eperm, post_eperm;

  // --- SMEM: smem layout M: offset bits (Vec, Bank, Seg)
  std::vector<u64> sw_vec, sw_bank, sw_seg, sw_H, sw_C;
  int sm_v = 0;                               // |Vec|
  std::vector<int> vec_slot_ld, vec_slot_st;  // reg bit positions of Vec in L_ld / L_st
  // smem element offset contributed by each kernel hardware bit (M^{-1} ∘ L)
  std::vector<u64> smoff_ld, smoff_st;
  u64 smem_elems = 0;
  long predicted_wavefronts_st = -1, predicted_wavefronts_ld = -1, ideal_wavefronts = -1;
  // Shared-memory instruction of each side (Thm 5.1), chosen by left
  // division of M^{-1}∘L by the instruction's tile:
  //   SMI_VEC  vectorised st/ld.shared (tile id_n^{Reg,Off}),
  //   SMI_MAT  stmatrix / ldmatrix m8n8 b16 (tile id_k^{Reg,Off} × id_2^{Thr,Off},
  //            k = log2(4/w)): reg word bits + lanes 0,1 form a 16-byte row,
  //            lanes 2-4 address the 8 rows of a matrix,
  //   SMI_MATT the .trans forms (w = 2): lanes 2-4 form the row, (word bit, lane 0,
  //            lane 1) address the rows.
  // ld = the smem store through L_ld, st = the smem load through L_st.
  int smi_ld = 0, smi_st = 0;
  std::vector<int> mat_word_ld, mat_word_st;   // reg bits forming a matrix word (k of them)
  std::vector<int> mat_sel_ld, mat_sel_st;     // reg bits selecting the matrix (.x1/.x2/.x4)
  long smem_instr_st = 0, smem_instr_ld = 0;   // shared instructions per thread per tile

  int threads() const { return 32 << Wb; }
  int elems_per_thread() const { return 1 << R; }
};

struct ConvPlan {
  Layout A, B;          // original (local) layouts
  int w = 4;
  ll_class cls = LL_CLASS_NOOP;   // the paper's class of A -> B
  int exec = EXEC_NOOP;
  std::vector<u64> Q;   // pull map: dst bit k -> src packed index (A^+ ∘ B, adjusted)
  u64 src_elems = 0, dst_elems = 0;
  TilePlan tile;
  // DEVICE plans (pack -> all-to-all -> unpack)
  int dev_bits = 0;
  size_t workspace_bytes = 0;
  ll_comm* comm = nullptr;
  std::unique_ptr<ConvPlan> pack, unpack;   // local stages of a DEVICE plan (null = identity)
  u64 chunk_elems = 0;                      // elements exchanged with every peer
  // Partial exchanges (dev bits shared by A and B): 2^xk chunks per
  // rank.  Send chunk j of rank r goes to rank (XOR of send_jcol over j's bits) ^ (XOR
  // of send_rcol over r's bits); recv chunk i of rank r comes from the analogous rank.
  int xk = 0;
  std::vector<uint32_t> send_jcol, send_rcol, recv_icol, recv_rcol;
  int send_peer(u64 j, int r) const {
    uint32_t q = 0;
    for (size_t b = 0; b < send_jcol.size(); ++b) if ((j >> b) & 1) q ^= send_jcol[b];
    for (size_t b = 0; b < send_rcol.size(); ++b) if ((r >> b) & 1) q ^= send_rcol[b];
    return int(q);
  }
  int recv_peer(u64 i, int r) const {
    uint32_t q = 0;
    for (size_t b = 0; b < recv_icol.size(); ++b) if ((i >> b) & 1) q ^= recv_icol[b];
    for (size_t b = 0; b < recv_rcol.size(); ++b) if ((r >> b) & 1) q ^= recv_rcol[b];
    return int(q);
  }
  int nranks = 1;
  u64 local_elems = 0;
  // DEVICE plans executed as peer stores (§8(f) N4): `fused` is one tile plan over the
  // global packed index space whose grid bits carrying the src dev bits come last;
  // rank r runs tiles [0, rank_tiles) with tile0 = r * rank_tiles.
  int exchange = 0;                         // LL_EXCHANGE_COLLECTIVE / LL_EXCHANGE_PEER
  std::unique_ptr<ConvPlan> fused;
  u64 rank_tiles = 0;
  int peer_shift = -1;    // >= 0: this tile plan is a peer kernel; log2 local elements
  bool peer_reg = false;  // a dst register / replica bit crosses ranks
  std::string tune_json;   // ll_plan_autotune: the candidates and their times (describe)
  std::string source;   // specialised kernel source (EXEC_TILE)
  std::string kernel_key;
  void* kernel = nullptr;   // cudaKernel_t once loaded
  int smem_bytes = 0;
  std::mutex mu;
};

std::unique_ptr<ConvPlan> plan_convert(const Layout& A, const Layout& B, int w, const ll_plan_opts* opts,
                                       u64 grid_only_src = 0);
Layout atomize(const Layout& L);   // 8-byte elements as pairs of 4-byte atoms (capi.cpp)
int num_sms();
void check_cuda(cudaError_t e, const char* what);
void launch_kernel(void* kernel, unsigned grid, unsigned block, void** args, size_t smem, cudaStream_t st,
                   const char* what);
// host mirror of LLPeers (ll_kernels.cuh): kernel parameter of the peer tile kernel
struct LLPeersHost { void* dst[64]; };
std::string describe(const ConvPlan& P);

struct GatherPlan {
  Layout L;
  int axis = 0, w = 4;
  int exec = EXEC_TILE;
  int sigma = SIGMA_COALESCED;
  int R = 0, Wb = 0, v = 0;
  int K_bits = 0;          // in-tile axis bits (K = 1 << K_bits)
  std::vector<int> hw_bit; // kernel bit -> packed bit (same for src, idx, dst)
  std::vector<u64> lcol;   // kernel bit -> logical column
  std::vector<int> grid_bit;
  // axis bit t (0..K_bits-1): position in the kernel: reg bit or lane bit (-1)
  std::vector<int> axis_reg_pos, axis_lane_pos;
  std::vector<int> axis_of_reg;  // kernel reg bit -> axis bit index or -1
  std::vector<int> axis_of_lane;
  int cand_bits = 0;       // |L_Reg^axis| in the kernel layout
  bool smem = false;       // shared-memory gather (too many shuffle candidates)
  std::vector<uint32_t> smoff;   // kernel bit -> smem element offset (logical tile order)
  uint32_t axmask = 0;           // smem offset bits of the in-tile axis bits
  std::vector<int> axpos;        // axis bit t -> smem offset bit
  int smem_bytes = 0;
  bool tma_store = false;  // outputs back into the stage, stored by cp.async.bulk
  bool tma = false;        // stream the contiguous src / idx tiles with cp.async.bulk
  int stages = 0;
  std::string source;
  void* kernel = nullptr;
  std::mutex mu;
};
std::unique_ptr<GatherPlan> plan_gather(const Layout& L, int axis, int w, const ll_plan_opts* opts);

struct ReducePlan {
  Layout L;
  int axis = 0;
  int exec = EXEC_TILE;
  int sigma = SIGMA_COALESCED;
  int op = 0;                     // 0 sum, 1 max, 2 min (ll_plan_opts.reduce_op)
  int R = 0, Wb = 0, v = 0;
  std::vector<int> hw_bit;        // kernel bit -> packed bit of L (σ)
  std::vector<int> grid_bit;      // CTA index bit -> packed bit (non-duplicate block bits)
  // reduced kernel bits per level (ascending); the steps run in logical axis bit order:
  // axis_hw[t] = the kernel bit holding in-tile axis bit t
  std::vector<int> red_reg, red_lane, red_warp;
  std::vector<int> axis_hw;
  int shfl_per_thread = 0;
  std::vector<int> dup_bits;      // zero-column kernel bits (de-dup)
  std::vector<u64> out_col;       // per kernel bit: output flat offset (0 for reduced/dup)
  std::vector<u64> grid_out;      // per grid bit: output flat offset
  u64 out_elems = 0;
  bool tma = false;        // stage each contiguous CTA tile with cp.async.bulk (UBLKCP)
  int wred_bytes = 0;      // smem for the warp-level stage
  int stages = 0;          // TMA pipeline depth
  std::string source;
  void* kernel = nullptr;
  int smem_bytes = 0;
  std::mutex mu;
};
std::unique_ptr<ReducePlan> plan_reduce(const Layout& L, int axis, const ll_plan_opts* opts);

// ------------------------------------------------------------------ codegen / jit
std::string codegen_tile(const ConvPlan& P);
// In-tile inclusive scan along an axis ("reduction and scan operations"; §8(f)
// N3), fixed fp32 order = the bit-doubling recurrence of reading R-scan.
struct ScanPlan {
  Layout L;
  int axis = 0;
  int sigma = SIGMA_COALESCED;
  int op = 0;                  // 0 sum, 1 max, 2 min (ll_plan_opts.reduce_op)
  int R = 0, Wb = 0, v = 0;
  int K_bits = 0;
  std::vector<int> hw_bit;     // kernel bit -> packed bit (src and dst)
  std::vector<int> grid_bit;   // CTA index bit -> packed bit
  std::vector<int> axis_hw;    // logical axis bit t -> kernel bit (reg < R or lane)
  int shfl_per_thread = 0;     // shuffles per thread per tile
  bool tma = false;            // cp.async.bulk staging of the contiguous CTA tiles
  bool tma_store = false;      // results written back into the stage, stored by cp.async.bulk
  int stages = 0;
  int xs_bytes = 0;            // exchange buffer of the warp-crossing steps
  int smem_bytes = 0;
  std::string source;
  void* kernel = nullptr;
  std::mutex mu;
};
std::unique_ptr<ScanPlan> plan_scan(const Layout& L, int axis, const ll_plan_opts* opts);
std::string codegen_scan(const ScanPlan& P);
std::string codegen_gather(const GatherPlan& P);
std::string codegen_reduce(const ReducePlan& P);
// Compile (or fetch from cache) and return a cudaKernel_t for `source`.
void* jit_kernel(const std::string& source, const char* name);
const char* kernel_template();   // embedded ll_kernels.cuh

// ------------------------------------------------------------------ host simulation (tests)
void simulate_tile(const ConvPlan& P, const uint8_t* src, uint8_t* dst);

}  // namespace ll

struct ll_layout { ll::Layout L; };
struct ll_plan {
  int kind;   // 0 conv, 1 gather, 2 reduce, 3 scan
  std::unique_ptr<ll::ConvPlan> conv;
  ll::ConvPlan* borrowed = nullptr;          // sub-plan handles (DEVICE stages)
  std::unique_ptr<ll_plan> stage[2];         // pack / unpack views of a DEVICE plan
  std::unique_ptr<ll::GatherPlan> gather;
  std::unique_ptr<ll::ReducePlan> reduce;
  std::unique_ptr<ll::ScanPlan> scan;
  ll::ConvPlan& cp() const { return borrowed ? *borrowed : *conv; }
};
struct ll_comm {
  int nranks = 1, rank = 0;
  bool loopback = false;   // all ranks' slices in one process (tests); memcpy exchange
  void* nccl = nullptr;    // ncclComm_t
  // peer windows (N4): every rank's dst window and barrier-flag buffer, mapped into
  // this process (CUDA IPC over NVLink); empty unless created by ll_comm_create_peers
  std::vector<void*> peer_dst, peer_flags;
  size_t window_bytes = 0;
  std::atomic<unsigned> epoch{0};
};
