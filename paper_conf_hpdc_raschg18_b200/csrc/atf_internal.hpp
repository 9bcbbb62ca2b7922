// atf_internal.hpp — structures shared by the host planner (planner.cpp, api.cpp)
// and the sm_100a kernels (kernels.cu).  Plain-old-data only: the level program is
// passed to the kernels by value as a kernel parameter (constant bank).
#pragma once
#include <stddef.h>
#include <stdint.h>

#ifdef __CUDACC__
#define ATF_HD __host__ __device__ __forceinline__
#else
#define ATF_HD inline
#endif

namespace atf {

constexpr int kMaxLevels = 64;   // parameters per group (= ATF_MAX_PARAMS)
constexpr int kMaxSlots = 24;    // per-node int64 values (ancestor params + hoisted invariants)
constexpr int kMaxTerms = 8;     // top-level conjuncts evaluated per candidate
constexpr int kMaxCode = 448;    // device bytecode words per level (invariants + generic terms)
constexpr int kMaxStack = 16;
constexpr int kMaxGroups = 64;
constexpr int kQTableMax = 16384;  // largest quotient with a shared-memory divisibility magic

// Device bytecode = the ABI opcodes plus SLOT k (push per-node slot k).
constexpr int32_t OP_SLOT = 32;

// Candidate-dependent conjunct kinds ("atoms").
enum TermKind : int32_t {
  T_CMP = 1,      // (A * x) rel B                                  A, B per node
  T_DIVX = 2,     // x | n        i.e. n mod x == 0, x == 0 rejects      A = |n|
  T_MULX = 3,     // d | x        i.e. x mod d == 0 (d != 0: node gate)  A = |d|, B = magic(d)
  T_DIVPROD = 4,  // (a*x) | b    -> gate a != 0 && a | b;  x | (b/a)    A = |b/a|
  T_QDIV = 5,     // (num / x) | nb, quotient 0 or x == 0 rejects        A = |num|, B = |nb|
  T_GENERIC = 6,  // any other conjunct: interpreted per candidate (code_off/code_len)
};
// arithmetic width the planner proved sufficient (static interval analysis)
enum Variant : int32_t { V16 = 0, V32 = 1, V64 = 2 };
enum Rel : int32_t { R_EQ = 11, R_NE = 12, R_LT = 13, R_LE = 14, R_GT = 15, R_GE = 16 };

struct Term {
  int32_t kind, variant, rel;
  int32_t slot_a, slot_b;      // operand slots (meaning per kind)
  int32_t code_off, code_len;  // T_GENERIC
  int32_t use_qtable;          // T_QDIV V16: divisibility magic of the quotient from smem
};

// Operand of a term on the narrow fast path (expand_nfast): an ancestor value, a constant
// or the product of two ancestor values, read straight from the parent record.
enum NfKind : int16_t { NF_PV = 0, NF_CONST = 1, NF_PROD = 2 };
struct NfOp {
  int16_t kind, s1, s2, pad;
  int32_t c;     // NF_CONST value
  uint32_t cm;   // NF_CONST: ceil(2^32/|c|) mod 2^32 (divisor magic)
};

// Per-level program + geometry, passed by value to the expand kernel.
constexpr int kMaxSeg = 8;     // warp-tile kernel: candidate segments per node
struct LevelArgs {
  // frontier = level k-1 of this group (k == 0: a single empty root record)
  const uint32_t* parent_rec;
  uint64_t n_parents;
  // candidates = materialised range of the level's parameter
  const int32_t* cand;         // int64 parameter (reading #22): the positions 0..r-1 (cand64 below)
  const uint32_t* cand_magic;  // ceil(2^32/|x|) mod 2^32 per candidate (2^16 for x == 0), host-computed
  const uint32_t* cand_abs;    // |x| per candidate; both padded to a multiple of 128
  int32_t r;
  int32_t level;
  int32_t field_word, field_shift;  // where the child's range position goes
  // slots [0, n_pv): values of ancestor levels, decoded from the parent record
  int32_t n_pv;
  int32_t pv_word[kMaxSlots], pv_shift[kMaxSlots], pv_bits[kMaxSlots];
  const int32_t* pv_range[kMaxSlots];  // int64 ancestors: pv_range64 below
  // slots [n_pv, n_slots): hoisted node-invariant expressions (code[inv_off..+inv_len))
  int32_t n_slots;
  int16_t inv_off[kMaxSlots], inv_len[kMaxSlots];
  // node gates: slot values that must be nonzero (top-level invariant conjuncts)
  int32_t n_gates;
  int16_t gate_slot[kMaxTerms];
  int32_t n_terms;
  Term terms[kMaxTerms];
  int32_t need_slots_smem;  // a generic term reads slots per candidate
  void* masks;              // nfast: per-parent accept masks (pass 1 -> pass 2)
  int32_t mask_bytes;       // 1, 2, 4 or 8
  int32_t direct;           // warp-tile: tiny level written in place (look-back over <= 16 tiles)
  int32_t nf_ok;            // narrow fast path possible (no gates / generic terms / wide variants)
  NfOp nf_op[kMaxTerms][2];
  const uint32_t* pv_magic[kMaxSlots];  // divisor magics of each ancestor's range
  int32_t need_m64;         // some term needs the 64-bit candidate magic
  int32_t code[kMaxCode];
  // outputs
  uint32_t* child_rec;      // [f_k][W]
  uint64_t* csr;            // [n_parents + 1]
  unsigned long long* status;  // [n_tiles] decoupled look-back tile status
  unsigned int* tile_counter;
  unsigned long long* total_out;
  uint64_t child_cap;       // capacity of child_rec in records
  unsigned int* overflow_flag;
  // wide levels: children go to per-tile stash segments first (no cross-tile wait),
  // then level_emit_kernel copies them to their final positions
  uint32_t* stash;          // [stash_cap][W]
  uint64_t stash_cap;
  unsigned long long* stash_top;
  uint32_t* tile_total;     // [n_tiles] children per tile
  unsigned long long* tile_seg;  // [n_tiles] stash segment (records)
  const uint64_t* tile_base;     // [n_tiles + 1] exclusive scan of tile_total
  const uint32_t* piece_tile;    // [total >> piece_shift + 1] tile holding output record p << piece_shift
  int32_t piece_shift;           // level_emit_kernel's piece size (2^7 for small levels, else 2^kPieceShift)
  // geometry (host choose_geometry)
  int32_t kind;             // K_NARROW: one thread per frontier node, r <= 64 candidates each
                            // K_WIDE:   each thread owns cpt consecutive candidates of a chunk
  int32_t block, cpt;
  int32_t hot, hot_term;    // wide: HOT_* filter of term hot_term evaluated in the hot loop
  int32_t tile_nodes;       // frontier nodes per tile (wide: multiple of 4)
  int32_t chunk;            // wide: candidates per chunk (= block * cpt)
  int32_t rw, sw;           // wide: bitmap words per node (chunk/32), summary words (ceil(rw/32))
  int32_t qcap;             // wide: slow-path queue entries per tile
  int32_t nseg;             // warp-tile: candidate segments of 32*cpt per node (<= kMaxSeg)
  int32_t seg_on;           // warp-tile: the per-segment |x| bounds below are applied
  // warp-tile hot filter, per segment: min / max |x| over its candidates (0 / 0xffffffff
  // when a candidate is 0).  x | n with n != 0 needs |x| <= |n|, d | x with x != 0 needs
  // |x| >= |d|: a node quad outside a segment's bounds has no item there
  uint32_t seg_lo[kMaxSeg], seg_hi[kMaxSeg];
  unsigned long long* pairs_out;  // ATF_FLAG_TIMING: (node, candidate) pairs the hot loop tested
  int64_t n_chunks;         // candidate chunks per node (r > chunk); tile_nodes == 4 padded, 1 real
  uint64_t n_tiles;
  uint32_t qmax;            // T_QDIV table covers quotients [0, qmax]
  int32_t smem_bytes;
  // int64 parameters (reading #22), at the end so the int32 kernels' parameter layout is unchanged:
  // the level's own values (its cand holds positions; generic terms only) and the referenced
  // int64 ancestors' value tables (else null).  pv64_any: some pv_range64 is set (no hot filter,
  // the generic prologue).
  const int64_t* cand64;
  const int64_t* pv_range64[kMaxSlots];
  int32_t pv64_any;
};
enum KernelKind : int32_t { K_NARROW = 0, K_WIDE = 1, K_WTILE = 2, K_NFAST = 3 };

// Fused narrow tail (DESIGN.md §5 "Narrow tail"): the last nl (2..kMaxTail) levels of a group,
// every one a narrow fast level (nf_ok, 1 <= r <= 32), expanded from the frontier of level
// t0 - 1 in two launches: tail_count (per warp tile of 32 frontier nodes: the tile's node
// count at every tail level) and, after an exclusive scan of those tile counts per level,
// tail_emit (the same masks again; every level's records and CSR written at their final
// positions through per-warp shared-memory buffers).  No intermediate level is re-read.
constexpr int kMaxTail = 4;
constexpr int kTailWarps = 4;  // warps per CTA of tail_emit
struct TailArgs {
  int32_t nl;
  const uint32_t* parent_rec;  // frontier (level t0 - 1); nullptr at t0 == 0 (root)
  uint64_t n_parents;
  uint64_t n_tiles;            // ceil(n_parents / 32)
  uint32_t* tile_total;        // [nl][n_tiles] (tail_count)
  const uint64_t* tile_base;   // [nl][n_tiles + 1] exclusive scans of tile_total per level
  uint32_t* node_cnt;          // [nl][n_parents] per frontier node subtree counts (NVRTC kernels)
  uint64_t* csr[kMaxTail];     // csr[0]: CSR of the frontier level [n_parents + 1];
                               // csr[d] (d >= 1): CSR of tail level d - 1
  uint32_t* rec[kMaxTail];     // records of tail level d (tail_emit)
  int32_t buf_off[kMaxTail];   // tail_emit: per-warp shared-memory buffer of level d (bytes)
  int32_t warp_bytes;          // tail_emit: shared memory per warp
  LevelArgs lv[kMaxTail];      // the levels' programs (narrow fast atoms) and candidates
};
constexpr int kNfNPL = 4;  // narrow fast kernel: frontier nodes per lane (warp tile = 128 nodes)
constexpr int kWT = 32;        // warp-tile kernel: frontier nodes per warp tile (one per lane)
constexpr int kItemCap = 512;  // warp-tile kernel: items whose exact masks pass 1 keeps for the emit pass
constexpr int kPieceShift = 10;  // level_emit_kernel copies the level in pieces of 2^10 records
                                 // (2^7 for levels below 2^20 records: more warps on a small level)
// Hot-loop filter of the wide kernel: a superset test of one conjunct, 2 instructions per
// (node, candidate) pair (IMAD + ISETP.OR into a per-node predicate).
enum HotKind : int32_t {
  HOT_NONE = 0,  // no filter: every (node, candidate) is evaluated exactly ("dense")
  HOT_DIVX = 1,  // x | n   (T_DIVX / T_DIVPROD, V16): n * ceil(2^32/x) <= ceil(2^32/x) - 1
  HOT_MULX = 2,  // d | x   (T_MULX, V16):            x * ceil(2^32/d) <= ceil(2^32/d) - 1
};
constexpr uint32_t kHotSentinel = 65521;  // largest 16-bit prime: hot operand of rejected nodes

// Decode: index -> per-group digit (mixed radix, group 0 most significant) ->
// leaf record -> range positions -> values.
struct DecodeArgs {
  int32_t n_groups;
  int32_t n_params;
  uint64_t gsize[kMaxGroups];
  uint64_t gmagic[kMaxGroups];  // floor((2^64 - 1) / gsize) (0 if gsize == 0): mixed-radix division
  const uint32_t* leaves[kMaxGroups];
  int32_t words[kMaxGroups];
  int32_t lvl_begin[kMaxGroups + 1];   // levels of group g: [lvl_begin[g], lvl_begin[g+1])
  int16_t lvl_param[kMaxLevels];
  int16_t lvl_word[kMaxLevels], lvl_shift[kMaxLevels], lvl_bits[kMaxLevels];
  const int32_t* lvl_range[kMaxLevels];
  const int64_t* lvl_range64[kMaxLevels];  // int64 parameters' value tables (else null), reading #22
};

// Encode (inverse decode): configuration -> per-group leaf index by
// a top-down walk of each group's tree (value -> range position by binary search in the
// parameter's sorted value table, position -> child by binary search among the node's
// children, which are sorted by position).
struct EncodeArgs {
  int32_t n_groups;
  uint64_t gsize[kMaxGroups];
  int32_t lvl_begin[kMaxGroups + 1];
  int16_t lvl_param[kMaxLevels], lvl_word[kMaxLevels], lvl_shift[kMaxLevels], lvl_bits[kMaxLevels];
  int32_t lvl_words[kMaxLevels];         // record words of the level's group
  const uint32_t* lvl_rec[kMaxLevels];   // level records [n][words]
  const uint64_t* lvl_csr[kMaxLevels];   // CSR of level l into level l + 1 (null at the leaves)
  uint64_t lvl_n[kMaxLevels];
  const int32_t* lvl_sorted[kMaxLevels]; // the parameter's [sorted values r][their positions r]
  int32_t lvl_r[kMaxLevels];
  // per parameter (neighbour proposals)
  int32_t n_params;
  int32_t param_group[kMaxLevels];
  int32_t param_r[kMaxLevels];
  const int32_t* param_range[kMaxLevels];  // values in range order
};

// CLTune-style baseline (SURVEY.md §8(f) NEXT-4, P:183 / P:280): enumerate the FULL
// cartesian product and test every constraint of every tuple.
struct ProductArgs {
  int32_t n_params;
  int32_t r[kMaxLevels];
  const int32_t* range[kMaxLevels];
  int32_t prog_first[kMaxLevels], prog_count[kMaxLevels];  // the parameter's programs in `progs`
  const int32_t* progs;    // [n_progs][2] (offset, length) into `code`
  const int32_t* code;     // device bytecode, OP_SLOT j = value of parameter j
  uint64_t total;          // product of the r (< 2^64)
  uint64_t chunk;          // tuples per thread (odometer)
};

// Dynamic shared-memory layouts of the expand kernels (byte offsets; -1 = absent).
struct SmemLayout {
  int ctl, ok, rec, opa, opb, slots, hot, hot2, cnt, off, sum, bm, q, cx, cm, qtab, wtot, total;
};
ATF_HD int align16(int x) { return (x + 15) & ~15; }
ATF_HD SmemLayout expand_layout(const LevelArgs& a, int words) {
  SmemLayout L;
  const int tn = a.tile_nodes;
  const bool wide = a.kind == K_WIDE;
  const int nc = wide ? a.chunk : a.r;  // candidate table entries
  int o = 0;
  L.ctl = o; o += 64;
  const int cols = wide ? tn : a.block;  // narrow: one operand column per thread, reused
  L.ok = o; o = align16(o + 4 * cols);
  L.rec = o; o = align16(o + 4 * words * cols);
  L.opa = o; o = align16(o + 8 * a.n_terms * cols);
  L.opb = o; o = align16(o + 8 * a.n_terms * cols);
  if (a.need_slots_smem) { L.slots = o; o = align16(o + 8 * a.n_slots * cols); } else { L.slots = -1; }
  if (wide) {
    L.hot = o; o = align16(o + 4 * tn);
    L.hot2 = o; o = align16(o + 4 * tn);
    L.cnt = o; o = align16(o + 4 * tn);
    L.off = o; o = align16(o + 4 * tn);
    L.sum = o; o = align16(o + 4 * tn * a.sw);
    L.bm = o; o = align16(o + 4 * tn * a.rw);
    L.q = o; o = align16(o + 4 * a.qcap);
  } else {
    L.hot = L.hot2 = L.cnt = L.off = L.sum = L.bm = L.q = -1;
  }
  if (!wide) {  // the wide kernel reads candidates and magics from global (L1)
    L.cx = o; o = align16(o + 4 * (nc > 0 ? nc : 1));
    L.cm = o; o = align16(o + 4 * (nc > 0 ? nc : 1));
  } else {
    L.cx = L.cm = -1;
  }
  if (a.qmax > 0) { L.qtab = o; o = align16(o + 4 * ((int)a.qmax + 1)); } else { L.qtab = -1; }
  L.wtot = o; o = align16(o + 8 * 34);
  L.total = o;
  return L;
}

// Warp-tile kernel layout: a CTA-wide candidate table (hot operand per candidate,
// transposed [seg][c][lane] so that lane b's CPT candidates are conflict-free) and one
// private region per warp (its tile's records, gates, hot operands, item words, operands).
struct WarpLayout {
  int tab, qtab, warp0, wstride;            // CTA part; warp w's region at warp0 + w * wstride
  int rec, ok, hot, hot2, cnt, items, imask, icode, opa, opb, slots;  // offsets inside a warp region
  int total;
};
ATF_HD WarpLayout wtile_layout(const LevelArgs& a, int words) {
  WarpLayout L;
  int o = 0;
  if (a.hot != HOT_NONE) { L.tab = o; o = align16(o + 4 * a.nseg * 32 * a.cpt); } else { L.tab = -1; }
  if (a.qmax > 0) { L.qtab = o; o = align16(o + 4 * ((int)a.qmax + 1)); } else { L.qtab = -1; }
  L.warp0 = o;
  int w = 0;
  L.rec = w; w = align16(w + 4 * words * kWT);
  L.ok = w; w += 4 * kWT;
  L.hot = w; w += 4 * kWT;
  L.hot2 = w; w += 4 * kWT;
  L.cnt = w; w += 4 * kWT;
  L.items = w; w = align16(w + 4 * kWT * a.nseg);
  L.imask = w; w = align16(w + 4 * kItemCap);
  L.icode = w; w = align16(w + 2 * kItemCap);
  L.opa = w; w = align16(w + 8 * kWT * a.n_terms);
  L.opb = w; w = align16(w + 8 * kWT * a.n_terms);
  if (a.need_slots_smem) { L.slots = w; w = align16(w + 8 * kWT * a.n_slots); } else { L.slots = -1; }
  L.wstride = w;
  L.total = o + w * (a.block / 32);
  return L;
}

// ---- launch wrappers (kernels.cu) ------------------------------------------------
// All return a cudaError_t value as int (0 = success).
int launch_expand(const LevelArgs& a, int words, void* stream);
int expand_smem_bytes(const LevelArgs& a, int words);
int launch_level_emit(const LevelArgs& a, int words, void* stream);
int launch_nfast_emit(const LevelArgs& a, int words, void* stream);
int launch_tail_count(const TailArgs& t, int words, void* stream);
int launch_tail_emit(const TailArgs& t, int words, void* stream);
}  // namespace atf
#include <vector>
namespace atf {
// jit.cpp: level-specialised pass-1 kernel of narrow fast levels (NVRTC, sm_100a)
void* jit_nfast_kernel(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                       const std::vector<uint32_t>& cand_magics);
int jit_nfast_launch(void* kernel, const LevelArgs& a, void* stream);
}  // namespace atf
#include <string>
namespace atf {
std::string jit_nfast_source(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                             const std::vector<uint32_t>& cand_magics);
// jit.cpp: fused narrow tail, specialised count + emit kernels (nullptr if not covered / no NVRTC)
// (k0 = the tail's first group level, pv_level[d][s] = group level of slot s's ancestor at tail level d)
std::string jit_tail_source(const TailArgs& t, int words, const std::vector<std::vector<int32_t>>& cand_values,
                            const std::vector<std::vector<uint32_t>>& cand_magics, int k0,
                            const std::vector<std::vector<int>>& pv_level);
void* jit_tail_kernels(const TailArgs& t, int words, const std::vector<std::vector<int32_t>>& cand_values,
                       const std::vector<std::vector<uint32_t>>& cand_magics, int k0,
                       const std::vector<std::vector<int>>& pv_level);
int jit_tail_launch(void* handle, const TailArgs& t, bool emit, void* stream);
// jit.cpp: mid-width levels (nf_ok, 32 < r <= kWideJitMax), specialised exact-mask kernel
constexpr int kWideJitMax = 1024;
std::string jit_wide_source(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                            const std::vector<uint32_t>& cand_magics);
void* jit_wide_kernel(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                      const std::vector<uint32_t>& cand_magics);
int jit_wide_smem(int r, int words);
int jit_wide_launch(void* kernel, const LevelArgs& a, int words, void* stream);
// jit.cpp: batched decode of one generated space (A9), specialised (nullptr if NVRTC fails)
std::string jit_decode_source(const DecodeArgs& a);
void* jit_decode_kernel(const DecodeArgs& a);
int jit_decode_launch(void* kernel, const DecodeArgs& a, const uint64_t* idx, const uint64_t* digits, int64_t n,
                      int32_t* out, int64_t ld, unsigned int* bad, void* stream);
// out: int32 SoA, or int64 SoA when w64 (reading #22)
int launch_decode_indices(const DecodeArgs& a, const uint64_t* idx, int64_t n, void* out, int w64,
                          int64_t ld, unsigned int* bad_flag, void* stream);
int launch_decode_digits(const DecodeArgs& a, const uint64_t* digits, int64_t n, void* out, int w64,
                         int64_t ld, unsigned int* bad_flag, void* stream);
int launch_decode128(const DecodeArgs& a, const uint64_t* idx_lo, const uint64_t* idx_hi, uint64_t first_lo,
                     uint64_t first_hi, int64_t n, void* out, int w64, int64_t ld, unsigned int* bad, uint64_t S_lo,
                     uint64_t S_hi, void* stream);
int launch_scan_u32(const uint32_t* in, uint64_t* out, int64_t n, unsigned long long* status,
                    unsigned int* counter, void* stream, uint32_t* piece_tile = nullptr,
                    uint64_t piece_cap = 0, int piece_shift = kPieceShift);
// `batch` independent scans of n elements in one launch (see scan_kernel)
int launch_scan_u32_batch(const uint32_t* in, uint64_t* out, int64_t n, int batch, unsigned long long* status,
                          uint64_t status_stride, unsigned int* counter, void* stream);
int launch_add_offset(uint64_t* data, uint64_t n, uint64_t add, void* stream);
void jit_set_tail_stage(int bytes);  // test hook: tail emit staging bytes per warp (0: default)
void jit_set_tail_product(bool on);  // test hook: product-structured tails on (default) / off
bool jit_tail_product(void* handle);  // the compiled tail's count is product-structured
void jit_set_tail_leaf_direct(int mode);
void jit_set_wide_group(int n);  // test hook: atf_wide_jit superset group size (4 or 8)  // test hook: leaf pass writes global memory (0 / 1 / 2 auto)
int launch_host_gate(const unsigned int* flag, unsigned int v, void* stream);
int launch_dist_flag_set(unsigned long long* f, unsigned long long v, void* stream);
int launch_dist_flag_wait(const unsigned long long* f, unsigned long long v, unsigned long long* err, void* stream);
int launch_divisible16_check(unsigned long long* mismatches, void* stream);
int launch_encode(const EncodeArgs& a, const int32_t* vals, int64_t ld, int64_t n, uint64_t* digits, uint64_t* idx,
                  void* stream);
int launch_filter_product(const ProductArgs& a, unsigned long long* count, void* stream);
int launch_neighbors(const EncodeArgs& a, const int32_t* in, int64_t ld_in, int32_t* out, int64_t ld_out, int64_t n,
                     uint64_t seed, int max_tries, int32_t* moved, void* stream);

}  // namespace atf
