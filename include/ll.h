/*
 * ll.h — C ABI of the B200-native linear-layout conversion library (libll.so).
 *
 * The method is "Linear Layouts: Robust Code Generation of Efficient Tensor
 * Computation Using F2" (ASPLOS '26).  Citations "P:L" are line numbers of the
 * paper text, with the section / definition given.
 *
 * CONVENTIONS
 *  - A layout is a linear map over F2 from labelled input (hardware) bits to
 *    labelled output (logical) bits (Def 4.1).  Input dims are named
 *    "reg", "lane", "warp", "block", "dev" (distributed layouts, Def 4.10) or
 *    "offset", "dev" (memory layouts, Def 4.14); output dims carry any names.
 *  - Hardware flat index h: the input dims' bits concatenated in declaration
 *    order, the FIRST declared dim least significant (P:138, P:148 footnote).
 *  - Logical flat index: row-major over the output dims in declaration order,
 *    the LAST dim fastest ("j is the fastest moving dimension").
 *  - A buffer "packed in layout L" is a dense array of 2^{d_in} elements of
 *    elem_bytes each; position h holds the logical element L(h).  A "dev" input
 *    dim must be declared last; rank r holds the slice dev = r.
 *  - Conversion is the pull form of B^{-1} ∘ A: for every dst index
 *    h, dst[h] = src[h'] for a preimage h' with A(h') = B(h).  The planner picks
 *    h' = Q(h), Q = A^+ ∘ B with the slack-zero right inverse and
 *    the identity on dims where A and B agree.
 *  - Precondition: src is A-consistent (A(h1) = A(h2) ⇒ equal elements); this
 *    always holds for data written through a layout.
 *
 * OWNERSHIP AND ERRORS
 *  - Handles (ll_layout, ll_plan, ll_comm) are created by the *_create / ll_plan_*
 *    calls and freed by the matching *_destroy.  Layouts and plans are immutable;
 *    a plan copies what it needs, so layouts may be destroyed after planning.
 *  - Device pointers are caller-owned (e.g. torch tensors), must be 16-byte
 *    aligned and stay alive until the stream work completes.
 *  - Every call returns an ll_status; nothing throws across the ABI;
 *    ll_last_error() returns a thread-local detail string.
 *  - ll_convert / ll_gather / ll_reduce are asynchronous on `stream`, never
 *    allocate device memory and never synchronise; asynchronous faults surface
 *    at the caller's synchronisation as CUDA errors.  There is no CPU fallback:
 *    the device entry points return LL_ERR_CUDA when no usable GPU is present.
 *
 * ENVIRONMENT (debugging / test hooks, read at planning time)
 *  - LL_FORCE_CLASS=shuffle|smem: the executed exchange of conversion plans whose
 *    opts leave force_class automatic (-1).
 *  - LL_LOG=1: every conversion plan is printed (ll_plan_describe JSON) to stderr.
 *  - LL_JIT_CACHE=<dir>: the NVRTC cubin cache (default: in-tree .ll_jit_cache/).
 *  - LL_PDL=0: launch without programmatic dependent launch.
 *  - LL_PIPE=0|1|staged|bulk|bulkst, LL_MIN_BLOCKS=k: override ll_plan_opts.pipe / min_blocks.
 *  - LL_NOHOIST=0|1: opaque thread bases in tile kernels (keeps XOR-combined addresses
 *    inside the tile loop; default on for linear tiles only).
 *  - LL_LINEAR_BALANCE=0: linear CTA tiles (general invertible pull maps) take the
 *    widest store runs instead of the default balanced load/store run lengths.
 *  - LL_BCAST=0: broadcast targets store their low replica bits per thread instead of
 *    through the dst-order smem read-back (TilePlan::bcast).
 *  - LL_BCAST_CTA=1|0: CTA-class broadcast maps try the CTA-tiled broadcast before (1)
 *    or never (0) instead of after the XOR-copy tiles (default).
 *  - LL_SCAN_TMA_STORE=0|1, LL_GATHER_TMA_STORE=0|1: scan / gather outputs stored per
 *    thread (0) or through the stage by cp.async.bulk (1); default: bulk stores for
 *    launches of <= 4096 tiles.
 *  - LL_XOR_INVEC=0: XOR-copy tiles shrink the vector instead of permuting in registers.
 *  - LL_ISOLATE_SMEM=1: diagnostic smem-exchange-only tile kernels (no global traffic).
 *  - LL_GRID_PER_SM=k: cap tile-kernel grids at k CTAs per SM (persistent CTAs looping
 *    over tiles); default / 0: one CTA per tile.
 *  - LL_ST_HINT=wb: tile kernels store with the default write-back policy instead of
 *    st.global.cs (evict-first streaming).
 *  - LL_AUX_MIN_BLOCKS=k: gather / reduce / scan kernels compiled with
 *    __launch_bounds__(threads, k), 0 = none (experiment; default: 2 for scans without
 *    a shared-memory warp step, none otherwise — profiles/r02_sweep_families_aux_min_blocks.jsonl).
 *  - LL_CTA_RUNS=+1|-1: CTA-class permutation tiles take src runs one bit longer (+1)
 *    or shorter (-1) than the dst runs (experiment; default: equal run lengths).
 *  - LL_NCCL_LIB=<path>: the libnccl.so.2 dlopen'ed for DEVICE plans (the Python binding
 *    points it at torch's NCCL).
 *  Host entry points (planning, launches) are wrapped in NVTX ranges named after
 *  the call (ll_plan_convert, ll_convert, ll_gather, ll_reduce, ll_scan).
 */
#ifndef LL_H_
#define LL_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  LL_OK = 0,
  LL_ERR_INVALID_ARG = 1,
  LL_ERR_DIM_MISMATCH = 2,
  LL_ERR_NOT_SURJECTIVE = 3,
  LL_ERR_NOT_INVERTIBLE = 4,
  LL_ERR_NOT_DIVISIBLE = 5,
  LL_ERR_UNSUPPORTED = 6,
  LL_ERR_ALIAS = 7,
  LL_ERR_MISALIGNED = 8,
  LL_ERR_CUDA = 9,
  LL_ERR_NVRTC = 10,
  LL_ERR_NCCL = 11,
  LL_ERR_OOM = 12
} ll_status;

/* The paper's conversion classes (P:364-373 and the smem fallback P:391),
 * extended with the cross-CTA and cross-GPU levels of the north star. */
typedef enum {
  LL_CLASS_NOOP = 0,    /* A(h) = B(h) for all h ("equivalent layouts")   */
  LL_CLASS_REGPERM = 1, /* (B^{-1}∘A)_Reg is a register permutation  */
  LL_CLASS_SHUFFLE = 2, /* warp part is the identity: warp shuffles  */
  LL_CLASS_SMEM = 3,    /* shared-memory round trip with optimal swizzle */
  LL_CLASS_CTA = 4,     /* mixes block (or memory-offset) bits                   */
  LL_CLASS_DEVICE = 5   /* mixes device bits: pack -> all-to-all -> unpack       */
} ll_class;

/* How a DEVICE plan moves data between GPUs.
 *   COLLECTIVE: pack -> all-to-all (grouped ncclSend/ncclRecv) -> unpack.
 *   PEER: one tile kernel per rank loads its src tiles and stores 16-byte vectors
 *         straight into the receivers' dst windows (NVLink peer memory, CUDA IPC),
 *         between two flag barriers; needs ll_comm_create_peers (or a loopback comm).
 *   AUTO: PEER when the communicator has peer windows, else COLLECTIVE. */
typedef enum { LL_EXCHANGE_AUTO = 0, LL_EXCHANGE_COLLECTIVE = 1, LL_EXCHANGE_PEER = 2 } ll_exchange;

typedef struct ll_layout ll_layout;
typedef struct ll_plan ll_plan;
typedef struct ll_comm ll_comm;

/* A labelled dimension: name and log2 of its size. */
typedef struct {
  const char* name;
  int log2_size;
} ll_dim;

typedef struct {
  int force_class;      /* -1 = auto; else an ll_class to execute (SHUFFLE/SMEM) */
  int max_vec_bytes;    /* global-memory vector bound, default 16    */
  int sigma;            /* 0 = coalesced HBM access (default), 1 = faithful      */
  int tile_bytes;       /* target CTA tile bytes when folding/choosing tiles (0 = default);
                         * linear tiles also take it as their size cap (default 64 KiB);
                         * gather / reduce / scan: split the layout's CTA tile down to
                         * it (warp bits of independent rows become grid bits; 0 = keep) */
  int thread_bytes;     /* target bytes per thread (0 = default: in-CTA tiles 256,
                         * or 64 when the layout's own CTA tile is below tile_bytes
                         * and grid bits are folded in; cross-CTA tiles: the tile's
                         * bytes / 256, within [elem_bytes, 256])                  */
  int generic;          /* 1 = force the runtime-generic kernel                   */
  ll_comm* comm;        /* required for DEVICE plans                              */
  int exchange;         /* DEVICE plans: an ll_exchange (default AUTO)            */
  int smem_instr;       /* smem round trips (Thm 5.1): 0 = auto — stmatrix /
                         * ldmatrix where M^{-1}∘L is divisible by their tile and that
                         * widens the swizzle's vector; 1 = vectorised ld/st.shared only;
                         * 2 = prefer stmatrix / ldmatrix wherever their tile divides   */
  int reduce_op;        /* ll_plan_reduce: 0 = sum (default), 1 = max, 2 = min (fp32)   */
  int pipe;             /* smem-exchange tiles: 0 = auto (= off), 1 = off,
                         * 2 = software-pipelined (next tile's loads
                         * before this tile's smem reads and HBM stores), 3 = staged
                         * (the next two tiles' 16-byte src vectors streamed by
                         * cp.async into two raw smem stages; persistent grid; needs
                         * 16-byte load vectors and exchange + 2 tiles <= 227 KiB),
                         * 4 = bulk (CTA tile contiguous in src order: whole tiles by
                         * cp.async.bulk into 2-3 raw stages, mbarrier completion),
                         * 5 = bulk load + bulk store (the dst tile, contiguous in dst
                         * order, leaves by cp.async.bulk from a dst stage).
                         * ll_plan_reduce / ll_plan_scan: 0 = auto (reduce: TMA stages
                         * only for >= 64 KiB tiles with an axis bit on the warps;
                         * scan: direct loads),
                         * 1 = direct 16-byte loads, 4 = TMA stages (cp.async.bulk of
                         * the contiguous CTA tile), 5 = TMA stages and (scan) the
                         * result tile out by cp.async.bulk                          */
  int min_blocks;       /* tile kernels: resident CTAs per SM requested from ptxas
                         * (__launch_bounds__ minimum): 0 = auto (2 for linear tiles and
                         * for unpipelined shuffle / smem tiles of 256 bytes per thread
                         * with <= 8 warps, else none), -1 = none, k >= 1 = k         */
} ll_plan_opts;

/* Fill *opts with defaults (force_class = -1, max_vec_bytes = 16, ...). */
void ll_plan_opts_default(ll_plan_opts* opts);

/* ---------------------------------------------------------------- layouts --
 * ll_layout_create (row a1; Def 4.1, matrix form P:140-148).
 *   in[n_in], out[n_out]: dims (names, log2 sizes); in-dim names must be unique.
 *   bases: Σ_i in[i].log2_size rows × n_out int64 coordinates; row k is the
 *          output coordinate hit by input bit k (hardware flat order).  Each
 *          coordinate must be < 2^{out log2_size}.  Copied; caller keeps ownership.
 *   *L: new handle.  Errors: LL_ERR_INVALID_ARG (bad sizes/names, > 64 bits).   */
ll_status ll_layout_create(const ll_dim* in, int n_in, const ll_dim* out, int n_out,
                           const int64_t* bases, ll_layout** L);
void ll_layout_destroy(ll_layout* L);

/* Shape queries: numbers of dims / total bits, and a dim's name and log2 size. */
ll_status ll_layout_info(const ll_layout* L, int* n_in, int* n_out, int* d_in, int* d_out);
ll_status ll_layout_dim(const ll_layout* L, int is_out, int index, const char** name, int* log2_size);
/* bases: d_in × n_out int64 (same format as ll_layout_create). */
ll_status ll_layout_bases(const ll_layout* L, int64_t* bases);

/* Evaluate L on one hardware coordinate tuple: XOR of the columns of the set bits
 * (P:136-148).  in_coords[n_in] -> out_coords[n_out]. */
ll_status ll_layout_apply(const ll_layout* L, const int64_t* in_coords, int64_t* out_coords);

/* Predicates: surjective, injective (rank), distributed (Def 4.10),
 * memory (Def 4.14).  Any output pointer may be NULL. */
ll_status ll_layout_props(const ll_layout* L, int* surjective, int* injective,
                          int* distributed, int* memory);

/* Composition outer∘inner (Def 4.2): requires inner's output dims to
 * equal outer's input dims (names and sizes, same order); else DIM_MISMATCH. */
ll_status ll_compose(const ll_layout* outer, const ll_layout* inner, ll_layout** out);

/* Right inverse (Def 4.5): Gaussian elimination over F2, free
 * variables 0, pivots in ascending column order; equals the min-index
 * preimage.  The result maps L's output dims to L's input dims.  Exact inverse
 * when L is bijective.  Errors: LL_ERR_NOT_SURJECTIVE. */
ll_status ll_invert(const ll_layout* L, ll_layout** out);

/* Product L1 × L2 (Def 4.3), label-wise: same-named dims concatenate
 * with L1's bits low; L2's images are shifted above L1's range. */
ll_status ll_product(const ll_layout* L1, const ll_layout* L2, ll_layout** out);

/* Left division M /_l M1 (Def 4.4): M2 such that M = M1 × M2
 * label-wise, or LL_ERR_NOT_DIVISIBLE.  Used for SIMD tiles (Thm 5.1). */
ll_status ll_left_divide(const ll_layout* M, const ll_layout* M1, ll_layout** M2);

/* Basis of ker(L) as hardware flat indices (broadcast directions; zero columns of
 * distributed layouts).  hw_vectors has room for d_in entries;
 * *n receives the count. */
ll_status ll_kernel_basis(const ll_layout* L, int64_t* hw_vectors, int* n);

/* ---------------------------------------------------------------- families --
 * Layout families (§4.3).  Output dims are named "d0", "d1", ... (row-major, last
 * fastest); all sizes are powers of two, else LL_ERR_INVALID_ARG.
 *
 * ll_layout_blocked (Prop 4.6 / 9.1): rank-`rank` tensor of
 *   `shape`; sizePerThread / threadsPerWarp / warpsPerCTA per dim; order[0] is the
 *   fastest dim.  Registers take sizePerThread bits in order, then lanes, then warps;
 *   a CTA tile smaller than the shape repeats over further register bits (in order),
 *   a larger one broadcasts (zero columns).  Fig. 1 A is
 *   blocked([16,16],[2,2],[4,8],[2,1],[1,0]). */
ll_status ll_layout_blocked(int rank, const int* shape, const int* size_per_thread,
                            const int* threads_per_warp, const int* warps_per_cta,
                            const int* order, ll_layout** L);
/* ll_layout_mma_acc (Prop 4.7 / 9.2): the mma m16n8 / wgmma
 * accumulator tile of an M x N output: reg0 -> j0, lanes (j1, j2, i0, i1, i2),
 * reg1 -> i3; warps along M first, then N; n-repetitions, then m-repetitions
 * as further register bits. */
ll_status ll_layout_mma_acc(int M, int N, int warps_m, int warps_n, ll_layout** L);
/* ll_layout_mma_swizzle (Def 4.11, Prop 4.12): the memory layout
 * offset -> (i, j) of a 2^m x 2^n tile, matrix [[I_n, C], [0, I_m]] with
 * c_i = (vec·((2^i/per_phase) mod max_phase)) mod 2^n. */
ll_status ll_layout_mma_swizzle(int log2_rows, int log2_cols, int vec, int per_phase,
                                int max_phase, ll_layout** L);
/* ll_layout_mma_operand (Prop 4.7 / 9.2): input
 * operand of mma (m16n8kK) / wgmma for `bitwidth`-bit elements (8, 16, 32).
 *   is_rhs = 0: lhs, rows x cols = M x K:
 *     id^{Reg,1}_{log2(32/b)} x id^{Thr,1}_2 x id^{Thr,0}_3 x id^{Reg,0}_1 x id^{Reg,1}_1
 *   is_rhs = 1: rhs, rows x cols = K x N:
 *     id^{Reg,0}_{log2(32/b)} x id^{Thr,0}_2 x id^{Thr,1}_3 x id^{Reg,1}_1
 *   Repetitions over K, then over the other dim, become register bits.  warps_m /
 *   warps_n split M / N; the operand's copies over the other dim's warps broadcast
 *   (zero columns).  wgmma's lhs is warps_m = 4 (id^{Wrp,0}_2). */
ll_status ll_layout_mma_operand(int is_rhs, int rows, int cols, int bitwidth, int warps_m,
                                int warps_n, ll_layout** L);
/* ll_layout_tmem_32x32b: the registers of a warpgroup after tcgen05.ld.32x32b from a
 * 128 x N fp32 TMEM accumulator (Blackwell tensor memory): thread t of warp w
 * holds row 32w + t, register r holds column r. */
ll_status ll_layout_tmem_32x32b(int M, int N, ll_layout** L);
/* ll_layout_tmem: the registers of a warpgroup after loading a 128 x N fp32 TMEM
 * accumulator with tcgen05.ld.sync.aligned.<shape>.x<num>.b32,
 * shape = "32x32b", "16x64b", "16x128b" or "16x256b" (TMEM lane = row d0, 32-bit TMEM
 * column = column d1; warp w owns lanes [32w, 32w+32)).  Per warp and x1 load:
 *   32x32b : thread -> row bits 0-4
 *   16x64b : thread bits -> (row 3, col 0, row 0, row 1, row 2)
 *   16x128b: thread bits -> (col 0, col 1, row 0-2); register -> row 3
 *   16x256b: thread bits -> (col 1, col 2, row 0-2); registers -> (col 0, row 3)
 * .x<num> repetitions along the columns are the next register bits; the 16-lane shapes
 * take a second load 16 lanes down (next register bit -> row 4); warps -> rows 5, 6.
 * Matches the CUTLASS SM100 TMEM_LOAD copy traits; tcgen05.st.<shape> takes its
 * registers in the same fragment (the TMEM_STORE traits reuse the load's thread and
 * value layouts), so the same layout describes an epilogue's TMEM store.
 * Errors: INVALID_ARG (M != 128,
 * unknown shape, N below one x1 load).  *L is owned by the caller (ll_layout_destroy). */
ll_status ll_layout_tmem(const char* shape, int M, int N, ll_layout** L);
/* ll_layout_contiguity (§5.1 "Contiguous elements"): the number of
 * elements each thread can move with one vector instruction — the largest u with
 * L^{-1}_Reg(i) = i for all i < u (leading register bits mapping in order to the
 * lowest logical bits, across dimensions), capped at max_vec_bytes (default 16 =
 * v4.b32). */
ll_status ll_layout_contiguity(const ll_layout* L, int elem_bytes, int max_vec_bytes, int* elems);
/* ll_layout_slice (Prop 4.8): drop logical dim `dim` (the result stays
 * surjective and may gain zero columns, Remark P:224). */
ll_status ll_layout_slice(const ll_layout* L, int dim, ll_layout** out);

/* ---------------------------------------------------------------- conversion --
 * ll_plan_convert (rows a2-a4, a6-a9).  Host only.
 *   A, B: same output dims; A surjective.  elem_bytes in {1, 2, 4, 8}.
 *   opts: NULL for defaults.  Computes Q = A^+ ∘ B, the paper's class (lowest
 *   hardware level Q must cross), and an execution plan: NOOP (a streaming copy
 *   kernel; nothing when src == dst), a
 *   specialised sm_100a tile kernel (register permutation / warp shuffles /
 *   swizzled smem round trip / cross-CTA tiled exchange), the runtime-generic
 *   kernel (broadcast and non-permutation maps), or DEVICE (pack, all-to-all over
 *   NVLink, unpack; needs opts->comm).  The specialised kernel is compiled with
 *   NVRTC for sm_100a on first use (cached on disk).
 *   Errors: DIM_MISMATCH, NOT_SURJECTIVE, INVALID_ARG, UNSUPPORTED. */
ll_status ll_plan_convert(const ll_layout* A, const ll_layout* B, int elem_bytes,
                          const ll_plan_opts* opts, ll_plan** plan);
ll_status ll_plan_class(const ll_plan* plan, ll_class* cls);
/* Workspace needed by ll_convert (> 0 only for DEVICE plans). */
ll_status ll_plan_workspace_bytes(const ll_plan* plan, size_t* bytes);
/* Bytes of each caller buffer the plan's execution call reads or writes (this rank's
 * slice for DEVICE plans): src and dst of ll_convert / ll_gather / ll_reduce / ll_scan
 * (2^{d_in} elements of the layout, §8(b) storage convention; ll_reduce's dst is
 * ll_plan_reduce_out_elems floats) and the int32 idx of ll_gather (0 for other kinds).
 * The execution calls take bare pointers: callers (the Python binding) check their
 * buffers against these sizes before launching.  Any out pointer may be NULL.
 * Errors: INVALID_ARG (null plan). */
ll_status ll_plan_buffer_bytes(const ll_plan* plan, size_t* src_bytes, size_t* dst_bytes, size_t* idx_bytes);
/* JSON description: class, executed exchange, V/I/E/F/G/R, swizzle columns,
 * rounds, predicted wavefronts, the smem instruction of each side (Thm 5.1:
 * "smem_store" / "smem_load", e.g. "stmatrix.m8n8.x4.b16", "ld.shared.v4.b32") and
 * their counts per thread per tile, launch geometry.  Truncates to cap bytes. */
ll_status ll_plan_describe(const ll_plan* plan, char* json, size_t cap);
/* Specialised CUDA source of the plan's kernel (empty if none). */
ll_status ll_plan_source(const ll_plan* plan, char* buf, size_t cap, size_t* needed);
/* Compile/load the plan's kernel now (otherwise done by the first launch). */
ll_status ll_plan_prepare(ll_plan* plan);
void ll_plan_destroy(ll_plan* plan);

/* ll_convert (rows a5-a10): dst[h] = src[Q(h)] on `stream` (a cudaStream_t).
 *   src: device buffer packed in A (2^{A.d_in} elements, local slice for dev);
 *   dst: device buffer packed in B; must not overlap src (LL_ERR_ALIAS), except
 *   that a NOOP plan accepts dst == src (in place: nothing runs); 16-byte aligned
 *   (LL_ERR_MISALIGNED).
 *   workspace: NULL unless ll_plan_workspace_bytes > 0.
 *   DEVICE plans are collective: every rank calls with the same plan. */
ll_status ll_convert(const void* src, void* dst, void* workspace, const ll_plan* plan,
                     void* stream);

/* ll_convert_host: the same conversion end to end from HOST buffers (pinned for
 * overlap): the batch is split into chunks of whole CTA tiles, and each chunk runs
 * H2D copy -> ll_tile_kernel -> D2H copy on streams[c % n_streams], so that copies in
 * both directions and the kernels of different chunks overlap.
 *   dev_buf: caller-owned device scratch of dev_buf_bytes (split into n_streams slots;
 *   each slot must hold at least one tile of src and dst).  Asynchronous: the caller
 *   synchronises the streams.  Tile plans whose CTA grid is the top bits of both
 *   buffers, and NOOP plans; else LL_ERR_UNSUPPORTED. */
ll_status ll_convert_host(const void* src_host, void* dst_host, void* dev_buf, size_t dev_buf_bytes,
                          const ll_plan* plan, int n_streams, void* const* streams);

/* ll_plan_autotune: measured plan selection for (A, B).  Plans the conversion under
 * each candidate kernel decomposition — `base` (NULL = defaults), thread_bytes 64 /
 * 128 / 256 when base leaves it 0, each also with a forced smem exchange when base
 * does not force a class, and each also with smem_instr = 1 (vectorised ld/st.shared
 * only) when base leaves it 0 (automatic stmatrix / ldmatrix) — compiles every distinct kernel, runs it `iters` times
 * (default 10) on the caller's src / dst (device buffers as for ll_convert; dst is
 * overwritten) on `stream`, and returns the fastest plan; describe lists the
 * candidates and their times ("autotune").  Synchronises `stream`.  Plans without a
 * tile kernel (NOOP, generic, DEVICE) are returned untuned.  Errors as
 * ll_plan_convert, plus LL_ERR_CUDA. */
ll_status ll_plan_autotune(const ll_layout* A, const ll_layout* B, int elem_bytes, const ll_plan_opts* base,
                           const void* src, void* dst, void* stream, int iters, ll_plan** plan);

/* ---------------------------------------------------------------- gather --
 * ll_plan_gather (row a11; §5.5).  src, idx and dst share layout L
 * (P:430).  Along logical dim `axis`, K = 2^(non-block axis bits of L); these
 * must be the low bits of the axis coordinate.  out[x] = src[x with the axis
 * coordinate's low bits replaced by idx[x] & (K-1)] (take_along_axis inside each
 * tile; out-of-range indices are masked).  Warp shuffles when
 * L_Wrp^axis = 0 and at most 2 candidate registers remain, else a
 * shared-memory gather over the staged CTA tile (any axis placement; the P:519
 * crossover); opts->force_class SHUFFLE / SMEM selects one (SHUFFLE with warp axis
 * bits: LL_ERR_UNSUPPORTED).  Direct 16-byte loads with opts->thread_bytes (default
 * 32) bytes of data per thread (non-axis register bits become warps); opts->pipe = 4
 * / 5 stages the src and idx tiles by cp.async.bulk (TMA) instead (5: and the dst tile
 * leaves by cp.async.bulk). */
ll_status ll_plan_gather(const ll_layout* L, int axis, int elem_bytes,
                         const ll_plan_opts* opts, ll_plan** plan);
/* src, dst: packed in L; idx: int32 packed in L. */
ll_status ll_gather(const void* src, const int32_t* idx, void* dst, const ll_plan* plan,
                    void* stream);

/* ---------------------------------------------------------------- reduce --
 * ll_plan_reduce (row a12; Table 4).  Sum (fp32; or max / min
 * with opts->reduce_op = 1 / 2) along logical dim `axis` over the non-block axis
 * bits of L (within each CTA tile; they must be the low bits of the axis
 * coordinate).  The fp32 order is fixed in logical coordinates (reading R-reduce,
 * DESIGN.md §3): for in-tile axis bit t = 0, 1, ... ascending, v <- v(t = 0) +
 * v(t = 1), round to nearest — the recursive pairwise sum, independent of L and of
 * every plan option.  Each step is a register add, a shfl.bfly or a shared-memory
 * step, whichever level of the kernel layout holds bit t; broadcast (zero-column)
 * bits are skipped, each output is written once.  LL_ERR_INVALID_ARG for another
 * reduce_op; LL_ERR_UNSUPPORTED when L is not distributed (Def 4.10). */
ll_status ll_plan_reduce(const ll_layout* L, int axis, const ll_plan_opts* opts, ll_plan** plan);
/* Number of output elements. */
ll_status ll_plan_reduce_out_elems(const ll_plan* plan, size_t* n);
/* src: fp32 packed in L; dst: fp32 logical row-major with the axis replaced by
 * its block part (one write per element). */
ll_status ll_reduce(const float* src, float* dst, const ll_plan* plan, void* stream);

/* ---------------------------------------------------------------- scan --
 * ll_plan_scan ("reduction and scan operations").  Inclusive
 * prefix sum (fp32) along `axis` inside each CTA tile of L (the in-tile axis bits are
 * the low bits of the axis coordinate, as for gather / reduce; each tile's scan starts
 * from zero).  The fp32 order is fixed (reading R-scan): for axis bit t =
 * 0, 1, ..., an element whose axis bit t is set adds the value of the last element of
 * the lower half of its aligned 2^(t+1)-block.  L: a distributed layout (duplicated
 * positions, zero columns, each get the same value).  Steps over register bits are
 * register adds, over lane bits warp shuffles, over warp bits a shared-memory
 * exchange (LL_ERR_UNSUPPORTED when it exceeds shared memory).  opts->reduce_op = 1 / 2
 * gives the running max / min instead of the sum (same steps, exact). */
ll_status ll_plan_scan(const ll_layout* L, int axis, const ll_plan_opts* opts, ll_plan** plan);
/* src, dst: fp32 packed in L (same positions); must not overlap partially. */
ll_status ll_scan(const float* src, float* dst, const ll_plan* plan, void* stream);

/* ---------------------------------------------------------------- comm --
 * NCCL communicator for DEVICE plans: nccl_unique_id is the 128-byte
 * ncclUniqueId produced by rank 0 and broadcast by the caller (e.g. over a torch
 * process group).  NCCL is loaded with dlopen on first use (LL_ERR_NCCL if
 * absent). */
ll_status ll_comm_create(const void* nccl_unique_id, int nranks, int rank, ll_comm** comm);
ll_status ll_comm_get_unique_id(void* nccl_unique_id /* 128 bytes */);
/* Single-process loopback communicator of nranks (power of two) virtual ranks: the
 * src / dst / workspace buffers passed to ll_convert hold all ranks' slices back to
 * back, and the exchange is a set of device memcpys.  For tests of the DEVICE
 * decomposition on one GPU. */
ll_status ll_comm_create_loopback(int nranks, ll_comm** comm);
/* Failure detection: LL_ERR_NCCL (with ncclGetErrorString's text in ll_last_error)
 * when an NCCL communicator has recorded an asynchronous error
 * (ncclCommGetAsyncError); LL_OK otherwise and for loopback / peer communicators,
 * whose failures surface as CUDA errors.  ll_convert checks it after each exchange. */
ll_status ll_comm_check(const ll_comm* comm);
void ll_comm_destroy(ll_comm* comm);

/* Peer-window communicator (§8(f) N4, LL_EXCHANGE_PEER).  Every rank owns a dst
 * window (>= the local dst size; ll_convert's dst must be exactly this rank's
 * window) and a zero-initialised flag buffer of LL_PEER_FLAG_BYTES; both are
 * caller-owned device memory, shared with the other ranks through CUDA IPC
 * (ll_ipc_export / ll_ipc_import) and mapped into this process.
 *   dst_windows[q], flag_bufs[q]: rank q's buffers as addressed from this process
 *   (this rank's own: its local pointers).  nranks <= LL_MAX_PEERS, power of two.
 * Copied; the caller keeps the mappings alive until ll_comm_destroy.  ll_convert
 * on such a plan is collective and stream-ordered: entry barrier, one tile kernel,
 * exit barrier (flag barriers spin on the GPU; a peer that never arrives traps the
 * kernel after 30 s instead of hanging). */
#define LL_PEER_FLAG_BYTES 512
#define LL_MAX_PEERS 64
ll_status ll_comm_create_peers(int nranks, int rank, void* const* dst_windows, void* const* flag_bufs,
                               size_t window_bytes, ll_comm** comm);

/* CUDA IPC of caller-owned device allocations (any pointer inside a cudaMalloc'd
 * block, e.g. a torch tensor): export writes LL_IPC_HANDLE_BYTES (the block's
 * cudaIpcMemHandle_t plus the pointer's offset in it); import maps it in another
 * process (one mapping per block, reference counted) and returns the pointer;
 * close drops the reference. */
#define LL_IPC_HANDLE_BYTES 72
ll_status ll_ipc_export(const void* dev_ptr, void* handle);
ll_status ll_ipc_import(const void* handle, void** dev_ptr);
ll_status ll_ipc_close(void* dev_ptr);

/* The stages of a DEVICE plan: pack (src -> send layout, receiver
 * rank bits on top) and unpack (recv layout, source rank bits on top -> dst); NULL
 * when a stage is the identity.  Every rank exchanges chunk_elems elements with
 * every peer.  The stage handles are owned by `plan` (do not destroy them). */
ll_status ll_plan_device_stages(const ll_plan* plan, ll_plan** pack, ll_plan** unpack,
                                size_t* chunk_elems, int* nranks);
/* ll_plan_device_peers: the chunk routing of a collective DEVICE plan for `rank`
 * (SURVEY §8(e)(2)).  The pack stage leaves *nchunks (= 2^xk <= nranks) equal chunks of
 * ll_plan_device_stages' chunk_elems; send chunk j goes to rank send_peers[j], and recv
 * chunk i (the unpack stage's input) comes from rank recv_peers[i].  A full exchange has
 * nchunks = nranks; a partial one (dev bits shared by A and B) talks to fewer ranks.
 * send_peers / recv_peers: caller arrays of >= nranks ints, or NULL.
 * Errors: INVALID_ARG (not a collective DEVICE plan, rank out of range). */
ll_status ll_plan_device_peers(const ll_plan* plan, int rank, int* send_peers, int* recv_peers, int* nchunks);

/* ---------------------------------------------------------------- test hooks --
 * ll_plan_simulate: host emulation of a specialised tile plan's schedule (the
 * same tables the kernel is specialised with: load addresses, pre/post register
 * networks, shuffle rounds and source lanes, smem offsets).  For validating the
 * planner on machines without a GPU; never used by ll_convert.  src/dst are HOST
 * buffers.  DEVICE plans with the peer exchange simulate their fused tile plan on
 * all ranks' slices back to back (the loopback buffer convention).
 * LL_ERR_UNSUPPORTED for other non-tile plans. */
ll_status ll_plan_simulate(const ll_plan* plan, const void* src, void* dst);

/* ll_jit_precompile: NVRTC-compile the plan's kernel into the on-disk cubin cache
 * without loading it (works without a GPU; used by the build to pre-populate the
 * cache for the benchmark configurations). */
ll_status ll_jit_precompile(const ll_plan* plan);

const char* ll_last_error(void);
const char* ll_version(void);

#ifdef __cplusplus
}
#endif
#endif /* LL_H_ */
