// atfgen.cpp — host side of libatfgen: the C ABI (include/atfgen.h), the planner
// (range materialisation, bytecode validation, static int64 interval analysis,
// group partition, hoisting + atom compilation of every level's constraint) and
// the generation driver (per-group arenas, one fused expand launch per level).
//
// Citations: P:n = PAPER.md line n; SURVEY.md §8 is the hot-path contract.
#include "../../include/atfgen.h"
#include "../../include/atfgen_test.h"

#include <cuda_runtime.h>

#include <unistd.h>

#include <algorithm>
#include <chrono>
#include <mutex>
#include <thread>
#include <array>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <functional>
#include <map>
#include <memory>
#include <numeric>
#include <string>
#include <vector>

#include "atf_internal.hpp"
#include <nvtx3/nvToolsExt.h>  // header-only NVTX3: ranges are free unless a profiler attaches

using namespace atf;

namespace {
// NVTX range for the lifetime of a scope (nsys / ncu --nvtx show the level rounds)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace
using i128 = __int128;
using u128 = unsigned __int128;

namespace {

enum State { BUILDING = 0, PLANNED = 1, GENERATED = 2, SHARDED = 3, FINAL_SHARD = 4 };

struct ParamDef {
  std::string name;
  // materialised range.  int32 parameter: the values.  int64 parameter (some value
  // outside int32, reading #22): the range positions 0..r-1, the values in values64; the
  // kernels map a position to its value through the int64 table (generic paths only).
  std::vector<int32_t> values;
  std::vector<int64_t> values64;
  bool v64 = false;
  std::vector<std::vector<int32_t>> programs;  // ANDed constraints
  int64_t vmin = 0, vmax = 0;
};

struct Iv {
  i128 lo, hi;
};
const i128 I64MIN = (i128)INT64_MIN, I64MAX = (i128)INT64_MAX;
bool fits64(const Iv& v) { return v.lo >= I64MIN && v.hi <= I64MAX; }
i128 absmax(const Iv& v) {
  i128 a = v.lo < 0 ? -v.lo : v.lo, b = v.hi < 0 ? -v.hi : v.hi;
  return a > b ? a : b;
}

struct ENode {
  int op = 0;
  int a = -1, b = -1;
  int64_t k = 0;  // PARAM id / CONST value
  bool var = false;
  Iv iv{0, 0};
  std::string key;
};

struct LevelPlan {
  int param = -1;
  int r = 0;
  int field_word = 0, field_shift = 0, field_bits = 0;
  LevelArgs proto;           // program part only
  std::vector<int> pv_param; // parameter id per ancestor slot
  double cost = 0;           // algorithmic int ops per candidate evaluation (roofline)
  bool generic = false;
  std::string desc;
  void* jit = nullptr;       // NVRTC-specialised narrow kernel (jit.cpp), if any
  void* wide_jit = nullptr;  // NVRTC-specialised mid-width kernel (jit.cpp), if any
  bool wide_jit_tried = false;
  int seg_cpt = -1;          // cpt the cached warp-tile segment bounds were computed for
  uint32_t seg_lo[kMaxSeg], seg_hi[kMaxSeg];
  bool jit_tried = false;
};

struct GroupPlan {
  std::vector<int> members;
  int words = 1;
  std::vector<LevelPlan> levels;
  void* tail_jit = nullptr;   // NVRTC-specialised tail kernels (jit.cpp), if any
  int tail_jit_k0 = -1;       // tail start they were built for (-1: not tried)
  int tail_ext_k0 = -1;       // extended tail start tried (NVRTC only), and whether it compiled
  bool tail_ext_ok = false;
};

struct Chunk {
  char* p = nullptr;
  size_t size = 0, used = 0;
  bool has_ipc = false;  // ipc handle exported (generate_dist)
  char ipc[64];
};

struct ReplayExpect { int round, g; uint64_t total; };  // a replayed level's expected total

struct LevelData {
  uint32_t* rec = nullptr;
  uint64_t* csr = nullptr;  // [n + 1], written when the next level is expanded
  uint64_t n = 0;
  uint64_t offset = 0;      // global index of rec[0] (shards)
  uint64_t csr_offset = 0;  // global index of the node whose CSR entry is csr[0] (shards)
  uint64_t csr_n = UINT64_MAX;  // csr entries - 1 (the nodes it covers); UINT64_MAX: the level's own nodes
  uint64_t evals = 0;
  float ms = -1.f;         // expand + scan + emit of the level (ATF_FLAG_TIMING)
  float expand_ms = -1.f;  // the expand kernel alone
  int32_t kernel = -1;     // KernelKind of the expand launch
  uint64_t pairs = 0;      // (node, candidate) pairs evaluated (ATF_FLAG_TIMING; = evals unless
                           // the warp-tile hot loop skipped segments by their |x| bounds)
  bool seg_skip = false;   // the level's hot loop applies the segment bounds
  int32_t cpt = 0, nseg = 0;  // warp-tile geometry of the level's last launch
  int32_t launches = 0;    // kernels launched for the level (re-runs included)
};

}  // namespace

// ---- balanced multi-GPU generation records (generate_dist)
struct DistDesc {       // where a rank's slice of a level (or its round-flag array) lives
  int64_t pid;          // owning process
  uint64_t base, off;   // allocation base (device pointer in the owner) and byte offset
  char handle[64];      // cudaIpcMemHandle_t of the allocation
};
struct DistGroup {      // per group, per round
  uint32_t nd, repl;    // levels completed this round (0, 1 or a tail's nl); replicated level
  uint64_t cnt[kMaxTail];
  DistDesc desc;        // records of the last completed level
};
constexpr int kDistMaxRounds = 256;

struct atf_space {
  atf_space_opts opts{};
  int state = BUILDING;
  std::string err;
  std::vector<ParamDef> params;
  std::vector<GroupPlan> groups;
  std::vector<int> group_of;
  // device state
  bool dev_ready = false;
  std::vector<int32_t*> d_range;
  std::vector<const int64_t*> d_range64;  // int64 parameters' value tables (else null)
  std::vector<int32_t*> d_sorted;  // per parameter: [values sorted ascending][their positions] (encode)
  std::vector<std::vector<Chunk>> arena;  // per group
  std::vector<std::vector<LevelData>> data;
  std::vector<uint64_t> gsize;
  unsigned long long* d_status = nullptr;
  size_t status_cap = 0;
  // per group (levels of different groups in one round run concurrently, one stream each)
  struct GroupBufs {
    char* masks = nullptr;      // nfast accept masks
    size_t masks_cap = 0;
    char* scratch = nullptr;    // per-tile totals, segments, bases, scan state
    size_t scratch_cap = 0;
    uint32_t* stash = nullptr;  // wide levels: children in tile segments before the final copy
    size_t stash_cap = 0;       // bytes
    unsigned long long* status = nullptr;  // tiny wide levels: look-back tile status words
    size_t status_cap = 0;                 // entries
    char* pbuf = nullptr;                  // generate_dist: this rank's parent slice, assembled
    size_t pbuf_cap = 0;                   // from the ranks' level arrays (P2P copies)
    cudaStream_t stream = nullptr;
    cudaEvent_t fork = nullptr, join = nullptr;
    cudaEvent_t done = nullptr;  // run_levels_async: the group's level and its result copies finished
  };
  std::vector<GroupBufs> gb;
  // run_levels_async: pinned per-group result slots [total u64 | overflow u32 | pad | tail totals u64[4]]
  unsigned long long* h_pin = nullptr;
  uint64_t stash_hint = 0;     // records: exact size of the last level that overflowed
  unsigned int* d_counter = nullptr;     // [kMaxGroups] tile counters
  unsigned long long* d_totals = nullptr;  // [kMaxGroups]
  unsigned int* d_ovf = nullptr;         // [kMaxGroups]
  unsigned int* d_bad = nullptr;         // decode flag
  unsigned long long* d_pairs = nullptr;  // [kMaxGroups] hot-loop pairs tested (ATF_FLAG_TIMING)
  uint32_t* d_root = nullptr;            // 8 zero words
  unsigned long long* h_totals = nullptr;  // -> h_totals_v
  unsigned int* h_flags = nullptr;         // -> h_flags_v
  std::vector<unsigned int> h_ctl;          // [totals u64 x kMaxGroups | ovf u32 x kMaxGroups]
  int32_t* d_table = nullptr;              // all parameter tables + scratch words (ensure_device)
  size_t table_bytes = 0;
  struct EvTriple { cudaEvent_t first = nullptr, mid = nullptr, second = nullptr; };
  std::vector<std::vector<EvTriple>> events;
  // fused narrow tails (one per group at most): count round -> emit round
  struct Tail {
    int k0 = -1, nl = 0;         // tail levels [k0, k0 + nl) of the group (k0 = -1: none)
    int phase = 0;               // 0 idle, 1 counted (totals known), 2 emitted
    TailArgs t;                  // kernel arguments (count and emit)
    uint64_t tot[kMaxTail] = {};  // node count of every tail level
  };
  std::vector<Tail> tails;
  // replay (DESIGN.md §5 "Steady state"): the level sizes of the last complete single-GPU
  // generation; the next generation of the space sizes every allocation and launch from them
  // and synchronises once, then verifies every level's total against them
  std::vector<std::vector<uint64_t>> replay_f;
  bool replay_ok = false;
  unsigned long long* d_replay = nullptr;  // per round: [totals u64 | ovf u32] of every group
  size_t replay_cap = 0;                   // rounds
  int replays = 0;                         // replays since the last level-by-level generation
  // the replay's launches captured once as a CUDA graph (DESIGN.md §5 "Steady state"): later
  // generations launch it whole; valid while no buffer it references moved (buf_epoch)
  cudaGraphExec_t graph_exec = nullptr;
  uint64_t graph_epoch = 0, buf_epoch = 0;
  bool capturing = false;
  cudaStream_t cap_stream = nullptr;
  cudaEvent_t cap_ev = nullptr;
  struct GraphSnap {  // host-side state of the captured generation
    std::vector<std::vector<LevelData>> data;
    std::vector<std::vector<size_t>> used;
    std::vector<Tail> tails;
    int rounds = 0;
    std::vector<ReplayExpect> expect;
    std::vector<int> tails_done;
  } gsnap;
  void* decode_jit = nullptr;   // specialised decoder of the current generation (jit.cpp)
  bool decode_jit_tried = false;
  // shards
  bool ipc_alloc = false;      // arena chunks from cudaMalloc (exported by CUDA IPC to peer ranks)
  struct PeerMap { int rank; char handle[64]; char* base; };
  std::vector<PeerMap> peers;  // opened IPC allocations of other ranks (generate_dist)
  int shard_rank = 0, shard_world = 1;
  // replayed balanced generation (DESIGN.md §6 "Steady state"): the last synchronous
  // generation's per-round all-gathers; once a generation with known sizes reproduced every
  // count, later ones queue all rounds without host synchronisation (device flags order the
  // cross-rank copies) and check everything once at the end
  struct DistLog {
    int world = 0, rank = -1;
    size_t G = 0;
    uint32_t flags = 0;
    std::vector<std::vector<DistGroup>> all;  // [round][world * G]
    std::vector<char> exchanged;               // [round]: an all-gather took place
    std::vector<DistDesc> flag_desc;           // [world]
    std::vector<uint64_t> cap_lo, cap_n;       // the group-to-rank assignment it was made with
    bool pure_ok = false;
  } dlog;
  std::vector<double> group_work;  // candidate pairs per group of the last generation (all ranks)
  unsigned long long* d_dflags = nullptr;  // [kDistMaxRounds] round flags | [1] wait timeout
  char dflags_ipc[64] = {};
  bool dflags_has_ipc = false;
  unsigned long long dist_epoch = 0;
  std::vector<cudaEvent_t> dist_ev;        // per round: [start, end] (ATF_FLAG_TIMING)
  std::vector<float> dist_round_ms;        // device time of this rank's rounds, last generation
  unsigned int* h_gate = nullptr;          // mapped host word releasing the timing gates
  unsigned int* d_gate = nullptr;
  unsigned int gate_v = 0;
  std::vector<int> shard_cut;  // per group: first level expanded on a slice (L = none)
};

// ---------------------------------------------------------------- helpers
static atf_status fail(atf_space* s, atf_status st, const char* fmt, ...) {
  if (s) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    s->err = buf;
  }
  return st;
}

#define CUDA_TRY(s, call)                                                                          \
  do {                                                                                             \
    cudaError_t e_ = (call);                                                                       \
    if (e_ != cudaSuccess) return fail((s), ATF_ERR_CUDA, "%s: %s", #call, cudaGetErrorString(e_)); \
  } while (0)

static void* dalloc(atf_space* s, size_t bytes) {
  if (bytes == 0) bytes = 16;
  void* p = nullptr;
  if (s->capturing) return nullptr;  // graph capture: no allocation (the capture is abandoned)
  s->buf_epoch++;
  if (s->ipc_alloc) {  // generate_dist: peers map the arena through CUDA IPC
    if (cudaMalloc(&p, bytes) != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
    }
  } else if (s->opts.alloc) {
    p = s->opts.alloc(bytes, s->opts.stream, s->opts.alloc_ctx);
  } else {
    if (cudaMallocAsync(&p, bytes, (cudaStream_t)s->opts.stream) != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
    }
  }
  return p;
}
static void dfree(atf_space* s, void* p, size_t bytes) {
  if (!p) return;
  s->buf_epoch++;
  if (s->ipc_alloc) {
    cudaStreamSynchronize((cudaStream_t)s->opts.stream);
    cudaFree(p);
  } else if (s->opts.alloc) {
    if (s->opts.free) s->opts.free(p, bytes, s->opts.stream, s->opts.alloc_ctx);
  } else {
    cudaFreeAsync(p, (cudaStream_t)s->opts.stream);
  }
}

static int bits_for(int64_t r) {
  int b = 0;
  while (((int64_t)1 << b) < r) b++;
  return b;
}

// ---------------------------------------------------------------- bytecode validation
// opcodes 1..21, PARAM j with j < self (reading #10), exactly one
// result, stack depth <= 16, <= 256 words.
static atf_status validate_program(atf_space* s, int self, const int32_t* code, int n) {
  if (n <= 0 || n > ATF_MAX_PROGRAM_WORDS) return fail(s, ATF_ERR_BYTECODE, "program length %d outside [1,256]", n);
  int sp = 0;
  for (int i = 0; i < n;) {
    int op = code[i];
    if (op == ATF_OP_X) { sp++; i++; }
    else if (op == ATF_OP_PARAM) {
      if (i + 1 >= n) return fail(s, ATF_ERR_BYTECODE, "PARAM without operand");
      int j = code[i + 1];
      if (j < 0 || j >= self)
        return fail(s, ATF_ERR_FORWARD_REF, "parameter %d references parameter %d (only earlier ones allowed)", self, j);
      sp++;
      i += 2;
    } else if (op == ATF_OP_CONST) {
      if (i + 2 >= n) return fail(s, ATF_ERR_BYTECODE, "CONST without operands");
      sp++;
      i += 3;
    } else if (op == ATF_OP_NOT) {
      if (sp < 1) return fail(s, ATF_ERR_BYTECODE, "stack underflow at word %d", i);
      i++;
    } else if (op >= ATF_OP_ADD && op <= ATF_OP_OR) {
      if (sp < 2) return fail(s, ATF_ERR_BYTECODE, "stack underflow at word %d", i);
      sp--;
      i++;
    } else {
      return fail(s, ATF_ERR_BYTECODE, "bad opcode %d at word %d", op, i);
    }
    if (sp > ATF_MAX_STACK) return fail(s, ATF_ERR_BYTECODE, "stack depth > %d", ATF_MAX_STACK);
  }
  if (sp != 1) return fail(s, ATF_ERR_BYTECODE, "program leaves %d items (must be 1)", sp);
  return ATF_OK;
}

// ---------------------------------------------------------------- expression trees
struct Tree {
  std::vector<ENode> nodes;
  int add(ENode n) {
    nodes.push_back(std::move(n));
    return (int)nodes.size() - 1;
  }
};

static const char* opname(int op) {
  static const char* names[] = {"?", "X", "PARAM", "CONST", "ADD", "SUB", "MUL", "DIV", "MOD", "MIN", "MAX", "EQ",
                                "NE", "LT", "LE", "GT", "GE", "DIVIDES", "MULOF", "AND", "OR", "NOT"};
  return (op >= 1 && op <= 21) ? names[op] : "?";
}

// interval of a binary op; false on possible int64 overflow (reading #9)
static bool binop_iv(int op, const Iv& a, const Iv& b, Iv& out) {
  auto mk = [&](i128 x, i128 y) { out = Iv{std::min(x, y), std::max(x, y)}; };
  switch (op) {
    case ATF_OP_ADD: out = Iv{a.lo + b.lo, a.hi + b.hi}; break;
    case ATF_OP_SUB: out = Iv{a.lo - b.hi, a.hi - b.lo}; break;
    case ATF_OP_MUL: {
      i128 c[4] = {a.lo * b.lo, a.lo * b.hi, a.hi * b.lo, a.hi * b.hi};
      out = Iv{*std::min_element(c, c + 4), *std::max_element(c, c + 4)};
      break;
    }
    case ATF_OP_DIV: {
      if (a.lo == I64MIN && b.lo <= -1 && b.hi >= -1) return false;  // INT64_MIN / -1
      if (a.lo >= 0 && b.lo > 0) mk(a.lo / b.hi, a.hi / b.lo);
      else { i128 m = absmax(a); out = Iv{-m, m}; }
      break;
    }
    case ATF_OP_MOD: {
      i128 mb = absmax(b) - 1;
      if (mb < 0) mb = 0;
      i128 ma = absmax(a);
      i128 m = std::min(ma, mb);
      if (a.lo >= 0) out = Iv{0, m};
      else if (a.hi <= 0) out = Iv{-m, 0};
      else out = Iv{-m, m};
      break;
    }
    case ATF_OP_MIN: out = Iv{std::min(a.lo, b.lo), std::min(a.hi, b.hi)}; break;
    case ATF_OP_MAX: out = Iv{std::max(a.lo, b.lo), std::max(a.hi, b.hi)}; break;
    default: out = Iv{0, 1}; break;
  }
  return fits64(out);
}

// Parse a validated program into the tree; returns the root node or -1 on overflow.
static int parse_program(const std::vector<int32_t>& code, const std::vector<ParamDef>& P, const Iv& xiv, Tree& t,
                         std::string* why) {
  std::vector<int> st;
  for (size_t i = 0; i < code.size();) {
    int op = code[i];
    ENode n;
    n.op = op;
    if (op == ATF_OP_X) {
      n.var = true;
      n.iv = xiv;
      n.key = "X";
      i++;
    } else if (op == ATF_OP_PARAM) {
      n.k = code[i + 1];
      n.iv = Iv{P[n.k].vmin, P[n.k].vmax};
      n.key = "P" + std::to_string(n.k);
      i += 2;
    } else if (op == ATF_OP_CONST) {
      n.k = (int64_t)(((uint64_t)(uint32_t)code[i + 2] << 32) | (uint64_t)(uint32_t)code[i + 1]);
      n.iv = Iv{n.k, n.k};
      n.key = "C" + std::to_string(n.k);
      i += 3;
    } else if (op == ATF_OP_NOT) {
      n.a = st.back();
      st.pop_back();
      n.var = t.nodes[n.a].var;
      n.iv = Iv{0, 1};
      n.key = "(" + t.nodes[n.a].key + " NOT)";
      i++;
    } else {
      n.b = st.back();
      st.pop_back();
      n.a = st.back();
      st.pop_back();
      const ENode &A = t.nodes[n.a], &B = t.nodes[n.b];
      n.var = A.var || B.var;
      if (!binop_iv(op, A.iv, B.iv, n.iv)) {
        if (why) *why = std::string("possible int64 overflow in ") + opname(op);
        return -1;
      }
      n.key = "(" + A.key + " " + B.key + " " + opname(op) + ")";
      i++;
    }
    st.push_back(t.add(std::move(n)));
  }
  return st.back();
}

// ---------------------------------------------------------------- level compiler
struct LevelCompiler {
  const std::vector<ParamDef>& P;
  Tree& t;
  LevelArgs& a;
  std::vector<int>& pv_param;
  std::map<std::string, int> slot_of_key;
  std::vector<int32_t> code;
  std::string err;
  int n_slots = 0;

  LevelCompiler(const std::vector<ParamDef>& P_, Tree& t_, LevelArgs& a_, std::vector<int>& pv)
      : P(P_), t(t_), a(a_), pv_param(pv) {}

  int pv_slot(int param) {
    for (size_t s = 0; s < pv_param.size(); s++)
      if (pv_param[s] == param) return (int)s;
    return -1;
  }
  // postfix code of a node; invariant subtrees become SLOT refs when `hoist`
  bool emit(int ni, std::vector<int32_t>& out, bool hoist) {
    const ENode& n = t.nodes[ni];
    if (hoist && !n.var) {
      int s = slot(ni);
      if (s < 0) return false;
      out.push_back(OP_SLOT);
      out.push_back(s);
      return true;
    }
    switch (n.op) {
      case ATF_OP_X: out.push_back(ATF_OP_X); return true;
      case ATF_OP_PARAM: out.push_back(OP_SLOT); out.push_back(pv_slot((int)n.k)); return true;
      case ATF_OP_CONST:
        out.push_back(ATF_OP_CONST);
        out.push_back((int32_t)(uint32_t)((uint64_t)n.k & 0xffffffffu));
        out.push_back((int32_t)(uint32_t)((uint64_t)n.k >> 32));
        return true;
      case ATF_OP_NOT:
        if (!emit(n.a, out, hoist)) return false;
        out.push_back(ATF_OP_NOT);
        return true;
      default:
        if (!emit(n.a, out, hoist) || !emit(n.b, out, hoist)) return false;
        out.push_back(n.op);
        return true;
    }
  }
  // slot holding the value of invariant node ni (deduplicated by structure)
  int slot(int ni) {
    const ENode& n = t.nodes[ni];
    if (n.op == ATF_OP_PARAM) return pv_slot((int)n.k);
    auto it = slot_of_key.find(n.key);
    if (it != slot_of_key.end()) return it->second;
    if (n_slots >= kMaxSlots) { err = "too many hoisted invariants"; return -1; }
    std::vector<int32_t> c;
    if (!emit(ni, c, false)) return -1;
    if (code.size() + c.size() > (size_t)kMaxCode) { err = "level program too long"; return -1; }
    int s = n_slots++;
    a.inv_off[s] = (int16_t)code.size();
    a.inv_len[s] = (int16_t)c.size();
    code.insert(code.end(), c.begin(), c.end());
    slot_of_key[n.key] = s;
    return s;
  }
  int mk_const(int64_t v) {
    ENode n;
    n.op = ATF_OP_CONST;
    n.k = v;
    n.iv = Iv{v, v};
    n.key = "C" + std::to_string(v);
    return t.add(n);
  }
  int mk_bin(int op, int x, int y) {  // invariant binary node; -1 on overflow
    ENode n;
    n.op = op;
    n.a = x;
    n.b = y;
    n.var = t.nodes[x].var || t.nodes[y].var;
    if (!binop_iv(op, t.nodes[x].iv, t.nodes[y].iv, n.iv)) return -1;
    n.key = "(" + t.nodes[x].key + " " + t.nodes[y].key + " " + opname(op) + ")";
    return t.add(n);
  }
};

static void flatten_and(const Tree& t, int ni, std::vector<int>& out) {
  const ENode& n = t.nodes[ni];
  if (n.op == ATF_OP_AND) {
    flatten_and(t, n.a, out);
    flatten_and(t, n.b, out);
  } else {
    out.push_back(ni);
  }
}

static int flip_rel(int rel) {
  switch (rel) {
    case R_LT: return R_GT;
    case R_GT: return R_LT;
    case R_LE: return R_GE;
    case R_GE: return R_LE;
    default: return rel;
  }
}

static const double kCost[] = {0, 2, 2, 2, 2, 6, 0};  // per TermKind (T_GENERIC: op count)

// Compile the constraint of level `lv` (parameter p) of a group.  Fills lp.proto's
// program part.  Returns ATF_OK or an error with message in *why.
static atf_status compile_level(const std::vector<ParamDef>& P, int p, const std::vector<int>& members, int lv,
                                const std::vector<int>& field_word, const std::vector<int>& field_shift,
                                const std::vector<int>& field_bits, bool generic_only, LevelPlan& lp,
                                std::string* why) {
  LevelArgs& a = lp.proto;
  std::memset(&a, 0, sizeof a);
  const ParamDef& pd = P[p];
  const Iv xiv{pd.vmin, pd.vmax};
  i128 xabs = absmax(xiv);
  Tree t;
  std::vector<int> roots;
  for (auto& code : pd.programs) {
    int root = parse_program(code, P, xiv, t, why);
    if (root < 0) return ATF_ERR_OVERFLOW;
    roots.push_back(root);
  }
  // ancestor slots: every parameter referenced by the level's programs
  std::vector<int> refs;
  for (auto& n : t.nodes)
    if (n.op == ATF_OP_PARAM && std::find(refs.begin(), refs.end(), (int)n.k) == refs.end()) refs.push_back((int)n.k);
  std::sort(refs.begin(), refs.end());
  if ((int)refs.size() > kMaxSlots) { *why = "too many referenced parameters"; return ATF_ERR_LIMIT; }
  lp.pv_param = refs;
  a.n_pv = (int)refs.size();
  for (int s = 0; s < a.n_pv; s++) {
    int l = (int)(std::find(members.begin(), members.end(), refs[s]) - members.begin());
    if (l >= lv) { *why = "internal: reference outside the group prefix"; return ATF_ERR_FORWARD_REF; }
    a.pv_word[s] = field_word[l];
    a.pv_shift[s] = field_shift[l];
    a.pv_bits[s] = field_bits[l];
  }
  LevelCompiler lc(P, t, a, lp.pv_param);
  lc.n_slots = a.n_pv;
  std::vector<Term> terms;
  std::vector<int> gates;
  std::vector<std::string> desc, gdesc;
  auto add_generic = [&](int ni) -> bool {
    std::vector<int32_t> c;
    if (!lc.emit(ni, c, !generic_only)) return false;
    Term T{};
    T.kind = T_GENERIC;
    T.code_off = (int)lc.code.size();
    T.code_len = (int)c.size();
    if (lc.code.size() + c.size() > (size_t)kMaxCode) { lc.err = "level program too long"; return false; }
    lc.code.insert(lc.code.end(), c.begin(), c.end());
    terms.push_back(T);
    desc.push_back("GENERIC" + std::string(" ") + t.nodes[ni].key);
    return true;
  };
  std::vector<int> conj;
  for (int root : roots) flatten_and(t, root, conj);
  if (generic_only) {
    // one interpreted term per program: no hoisting, no atoms (baseline path)
    for (int root : roots)
      if (!add_generic(root)) { *why = lc.err; return ATF_ERR_LIMIT; }
  } else {
    for (int ci : conj) {
      const ENode& n = t.nodes[ci];
      if (!n.var) {  // node-invariant conjunct -> node gate
        int s = lc.slot(ci);
        if (s < 0) { *why = lc.err; return ATF_ERR_LIMIT; }
        gates.push_back(s);
        gdesc.push_back("GATE " + n.key);
        continue;
      }
      Term T{};
      bool matched = false;
      auto isX = [&](int i) { return t.nodes[i].op == ATF_OP_X; };
      auto inv = [&](int i) { return !t.nodes[i].var; };
      // DIVIDES(d, m): d | m.  MULOF(m, d) is the same test with the same poison (d == 0).
      int d = -1, m = -1;
      if (n.op == ATF_OP_DIVIDES) { d = n.a; m = n.b; }
      if (n.op == ATF_OP_MULOF) { d = n.b; m = n.a; }
      if (d >= 0) {
        const ENode& D = t.nodes[d];
        if (isX(d) && inv(m)) {  // x | m
          T.kind = T_DIVX;
          T.slot_a = lc.slot(m);
          i128 nm = absmax(t.nodes[m].iv);
          T.variant = (xabs < 65536 && nm < 65536) ? V16 : (nm < ((i128)1 << 32) ? V32 : V64);
          matched = T.slot_a >= 0;
        } else if (inv(d) && isX(m)) {  // d | x
          T.kind = T_MULX;
          T.slot_a = lc.slot(d);
          i128 dm = absmax(D.iv);
          T.variant = (xabs < 65536 && dm < 65536) ? V16 : (dm < ((i128)1 << 32) ? V32 : V64);
          matched = T.slot_a >= 0;
        } else if (D.op == ATF_OP_MUL && inv(m) && ((isX(D.a) && inv(D.b)) || (inv(D.a) && isX(D.b)))) {
          // (a*x) | m  ->  gate a != 0 && a | m;  x | (m / a)
          int an = isX(D.a) ? D.b : D.a;
          T.kind = T_DIVPROD;
          T.slot_a = lc.slot(an);
          T.slot_b = lc.slot(m);
          i128 nm = absmax(t.nodes[m].iv);
          T.variant = (xabs < 65536 && nm < 65536) ? V16 : (nm < ((i128)1 << 32) ? V32 : V64);
          matched = T.slot_a >= 0 && T.slot_b >= 0;
        } else if (D.op == ATF_OP_DIV && inv(D.a) && isX(D.b) && inv(m)) {
          // (num / x) | m
          T.kind = T_QDIV;
          T.slot_a = lc.slot(D.a);
          T.slot_b = lc.slot(m);
          i128 nu = absmax(t.nodes[D.a].iv), nb = absmax(t.nodes[m].iv);
          if (xabs < 65536 && nu < 65536 && nb < 65536) {
            T.variant = V16;
            // the quotient's divisibility test divides inline (32-bit): QDIV is only reached
            // by survivors of the cheaper conjuncts, and a per-CTA magic table of the
            // quotients would cost shared memory that bounds the tile size
            T.use_qtable = 0;
          } else {
            T.variant = (nu < ((i128)1 << 32) && nb < ((i128)1 << 32)) ? V32 : V64;
          }
          matched = T.slot_a >= 0 && T.slot_b >= 0;
        }
      } else if (n.op >= ATF_OP_EQ && n.op <= ATF_OP_GE) {
        int vs = -1, is = -1, rel = n.op;
        if (t.nodes[n.a].var && inv(n.b)) { vs = n.a; is = n.b; }
        else if (inv(n.a) && t.nodes[n.b].var) { vs = n.b; is = n.a; rel = flip_rel(rel); }
        if (vs >= 0) {
          // affine side: x, a*x, x*a, x+c, c+x, x-c, c-x  ->  (m*x + c) rel v  ->  m*x rel v - c
          const ENode& V = t.nodes[vs];
          int mnode = -1, cnode = -1;
          bool neg_c = false;
          if (isX(vs)) { mnode = lc.mk_const(1); }
          else if (V.op == ATF_OP_MUL && isX(V.a) && inv(V.b)) { mnode = V.b; }
          else if (V.op == ATF_OP_MUL && inv(V.a) && isX(V.b)) { mnode = V.a; }
          else if (V.op == ATF_OP_ADD && isX(V.a) && inv(V.b)) { mnode = lc.mk_const(1); cnode = V.b; }
          else if (V.op == ATF_OP_ADD && inv(V.a) && isX(V.b)) { mnode = lc.mk_const(1); cnode = V.a; }
          else if (V.op == ATF_OP_SUB && isX(V.a) && inv(V.b)) { mnode = lc.mk_const(1); cnode = V.b; neg_c = true; }
          else if (V.op == ATF_OP_SUB && inv(V.a) && isX(V.b)) { mnode = lc.mk_const(-1); cnode = V.a; }
          if (mnode >= 0) {
            int vnode = is;
            if (cnode >= 0) vnode = lc.mk_bin(neg_c ? ATF_OP_ADD : ATF_OP_SUB, is, cnode);
            if (vnode >= 0) {
              Iv prod;
              bool ok = binop_iv(ATF_OP_MUL, t.nodes[mnode].iv, xiv, prod);
              if (ok) {
                T.kind = T_CMP;
                T.rel = rel;
                T.slot_a = lc.slot(mnode);
                T.slot_b = lc.slot(vnode);
                const Iv& vi = t.nodes[vnode].iv;
                bool f32 = prod.lo >= INT32_MIN && prod.hi <= INT32_MAX && vi.lo >= INT32_MIN && vi.hi <= INT32_MAX &&
                           t.nodes[mnode].iv.lo >= INT32_MIN && t.nodes[mnode].iv.hi <= INT32_MAX;
                T.variant = f32 ? V32 : V64;
                matched = T.slot_a >= 0 && T.slot_b >= 0;
              }
            }
          }
        }
      } else if (isX(ci)) {  // bare x as a conjunct: x != 0
        T.kind = T_CMP;
        T.rel = R_NE;
        T.slot_a = lc.slot(lc.mk_const(1));
        T.slot_b = lc.slot(lc.mk_const(0));
        T.variant = V32;
        matched = T.slot_a >= 0 && T.slot_b >= 0;
      }
      if (!lc.err.empty()) { *why = lc.err; return ATF_ERR_LIMIT; }
      if (matched) {
        terms.push_back(T);
        static const char* kn[] = {"?", "CMP", "DIVX", "MULX", "DIVPROD", "QDIV", "GENERIC"};
        static const char* vn[] = {"16", "32", "64"};
        desc.push_back(std::string(kn[T.kind]) + "/" + vn[T.variant] + " " + n.key);
      } else if (!add_generic(ci)) {
        *why = lc.err;
        return ATF_ERR_LIMIT;
      }
    }
  }
  // cheapest conjuncts first (top-level AND: order changes neither result nor poison-reject)
  std::vector<size_t> order(terms.size());
  std::iota(order.begin(), order.end(), 0);
  auto cost_of = [&](const Term& T) { return T.kind == T_GENERIC ? 10.0 + T.code_len : kCost[T.kind]; };
  std::stable_sort(order.begin(), order.end(), [&](size_t x, size_t y) { return cost_of(terms[x]) < cost_of(terms[y]); });
  if ((int)terms.size() > kMaxTerms) { *why = "too many conjuncts"; return ATF_ERR_LIMIT; }
  if ((int)gates.size() > kMaxTerms) { *why = "too many invariant conjuncts"; return ATF_ERR_LIMIT; }
  a.n_terms = (int)terms.size();
  lp.cost = 0;
  lp.generic = false;
  std::string d;
  for (size_t i = 0; i < order.size(); i++) {
    const Term& T = terms[order[i]];
    a.terms[i] = T;
    if (T.kind == T_GENERIC) {
      a.need_slots_smem = 1;
      lp.generic = true;
      int ops = 0;
      for (int w = T.code_off; w < T.code_off + T.code_len;) {
        int op = lc.code[w];
        ops++;
        w += (op == OP_SLOT) ? 2 : (op == ATF_OP_CONST ? 3 : 1);
      }
      lp.cost += ops;
    } else {
      lp.cost += kCost[T.kind];
    }
    if (T.kind == T_DIVX || T.kind == T_DIVPROD || T.kind == T_MULX || T.kind == T_QDIV)
      if (T.variant == V32) a.need_m64 = 1;
    d += (i ? " & " : "") + desc[order[i]];
  }
  if (a.n_terms > 1) lp.cost += a.n_terms - 1;  // the ANDs
  a.n_gates = (int)gates.size();
  for (size_t i = 0; i < gates.size(); i++) {
    a.gate_slot[i] = (int16_t)gates[i];
    d += std::string(d.empty() ? "" : " & ") + gdesc[i];
  }
  a.n_slots = lc.n_slots;
  if (lc.code.size() > (size_t)kMaxCode) { *why = "level program too long"; return ATF_ERR_LIMIT; }
  std::copy(lc.code.begin(), lc.code.end(), a.code);
  // narrow fast path (expand_nfast): no gates, every conjunct a 16-bit divisibility atom or a
  // 32-bit comparison whose operands are ancestor values, constants or ancestor products
  {
    auto opdesc = [&](int slot, NfOp& o) -> bool {
      o = NfOp{};
      if (slot < 0) return false;
      if (slot < a.n_pv) { o.kind = NF_PV; o.s1 = (int16_t)slot; return true; }
      const int32_t* c = a.code + a.inv_off[slot];
      const int len = a.inv_len[slot];
      if (len == 3 && c[0] == ATF_OP_CONST) {
        const int64_t v = (int64_t)(((uint64_t)(uint32_t)c[2] << 32) | (uint32_t)c[1]);
        if (v < INT32_MIN || v > INT32_MAX) return false;
        o.kind = NF_CONST;
        o.c = (int32_t)v;
        const uint32_t av = v < 0 ? 0u - (uint32_t)v : (uint32_t)v;
        o.cm = av > 1 ? 0xffffffffu / av + 1u : 0u;
        return true;
      }
      if (len == 5 && c[0] == OP_SLOT && c[2] == OP_SLOT && c[4] == ATF_OP_MUL && c[1] < a.n_pv && c[3] < a.n_pv) {
        o.kind = NF_PROD;
        o.s1 = (int16_t)c[1];
        o.s2 = (int16_t)c[3];
        return true;
      }
      return false;
    };
    bool ok = a.n_gates == 0 && !lp.generic;
    for (int r : lp.pv_param)
      if (P[r].v64) ok = false;  // the fast paths read int32 value tables only
    for (int t = 0; ok && t < a.n_terms; t++) {
      const Term& T = a.terms[t];
      switch (T.kind) {
        case T_DIVX: case T_MULX: ok = T.variant == V16 && opdesc(T.slot_a, a.nf_op[t][0]); break;
        case T_DIVPROD: case T_QDIV:
          ok = T.variant == V16 && !T.use_qtable && opdesc(T.slot_a, a.nf_op[t][0]) && opdesc(T.slot_b, a.nf_op[t][1]);
          break;
        case T_CMP: ok = T.variant == V32 && opdesc(T.slot_a, a.nf_op[t][0]) && opdesc(T.slot_b, a.nf_op[t][1]); break;
        default: ok = false;
      }
    }
    a.nf_ok = ok ? 1 : 0;
  }
  lp.desc = d.empty() ? "TRUE" : d;
  return ATF_OK;
}

// ---------------------------------------------------------------- planning
static atf_status plan(atf_space* s) {
  if (s->state != BUILDING) return ATF_OK;
  int n = (int)s->params.size();
  // groups: connected components of p -- q for every q referenced by p's constraints
  // (groups ordered by first member, members in declaration order)
  std::vector<int> parent(n);
  std::iota(parent.begin(), parent.end(), 0);
  std::function<int(int)> find = [&](int x) { return parent[x] == x ? x : parent[x] = find(parent[x]); };
  for (int p = 0; p < n; p++)
    for (auto& code : s->params[p].programs)
      for (size_t i = 0; i < code.size();) {
        int op = code[i];
        if (op == ATF_OP_PARAM) {
          int a = find(p), b = find(code[i + 1]);
          if (a != b) parent[std::max(a, b)] = std::min(a, b);
          i += 2;
        } else {
          i += (op == ATF_OP_CONST) ? 3 : 1;
        }
      }
  s->groups.clear();
  s->group_of.assign(n, -1);
  std::map<int, int> gid;
  for (int p = 0; p < n; p++) {
    int root = find(p);
    auto it = gid.find(root);
    if (it == gid.end()) {
      gid[root] = (int)s->groups.size();
      s->groups.push_back(GroupPlan{});
      it = gid.find(root);
    }
    s->groups[it->second].members.push_back(p);
    s->group_of[p] = it->second;
  }
  if ((int)s->groups.size() > kMaxGroups) return fail(s, ATF_ERR_LIMIT, "more than %d groups", kMaxGroups);
  for (auto& g : s->groups) {
    // record layout: each level's range position gets ceil(log2 r) bits; fields are
    // packed first-fit-decreasing into 32-bit words (no field straddles a word)
    size_t L = g.members.size();
    std::vector<int> fw(L, 0), fs(L, 0), fb(L, 0);
    for (size_t l = 0; l < L; l++) fb[l] = bits_for((int64_t)s->params[g.members[l]].values.size());
    std::vector<size_t> ord(L);
    std::iota(ord.begin(), ord.end(), 0);
    std::stable_sort(ord.begin(), ord.end(), [&](size_t x, size_t y) { return fb[x] > fb[y]; });
    std::vector<int> fill;
    for (size_t l : ord) {
      size_t w = 0;
      while (w < fill.size() && fill[w] + fb[l] > 32) w++;
      if (w == fill.size()) fill.push_back(0);
      fw[l] = (int)w;
      fs[l] = fb[l] ? fill[w] : 0;  // a 0-bit field (r <= 1) never shifts by 32
      fill[w] += fb[l];
    }
    int words = std::max<int>(1, (int)fill.size());
    if (words > 8) return fail(s, ATF_ERR_LIMIT, "group path record needs %d words (> 8)", words);
    g.words = words <= 1 ? 1 : words <= 2 ? 2 : words <= 4 ? 4 : 8;
    g.levels.clear();
    for (size_t l = 0; l < g.members.size(); l++) {
      LevelPlan lp;
      int p = g.members[l];
      lp.param = p;
      lp.r = (int)s->params[p].values.size();
      lp.field_word = fw[l];
      lp.field_shift = fs[l];
      lp.field_bits = fb[l];
      std::string why;
      // an int64 parameter's own level is interpreted in int64 (reading #22)
      atf_status st = compile_level(s->params, p, g.members, (int)l, fw, fs, fb,
                                    (s->opts.flags & ATF_FLAG_GENERIC_ONLY) != 0 || s->params[p].v64, lp, &why);
      if (st != ATF_OK) return fail(s, st, "parameter %s: %s", s->params[p].name.c_str(), why.c_str());
      lp.proto.level = (int)l;
      lp.proto.field_word = fw[l];
      lp.proto.field_shift = fs[l];
      g.levels.push_back(lp);
    }
  }
  s->state = PLANNED;
  return ATF_OK;
}

// ---------------------------------------------------------------- geometry
// r <= 64 -> narrow kernel (thread per node); otherwise the wide
// kernel with cpt candidates per thread, a hot filter when a conjunct allows one, and
// ~2^18 (node, candidate) pairs per tile.
// Tuning knobs with test hooks (atf_test_set_geometry): warp tiles per SM below which the
// warp-tile kernel halves its nodes per tile, and the pair count below which generate_dist
// replicates a level instead of distributing it.
static std::atomic<int> g_tiles_per_sm{256};
static std::atomic<int> g_repl_log2{28};
static std::atomic<int> g_direct_tiles{16};  // in-place (look-back) levels: at most this many warp tiles
static std::atomic<int> g_async_rounds{1};   // fresh spaces: per-group rounds without a barrier

static void choose_geometry(LevelArgs& a, int words, bool legacy_wide, bool seg_bounds = true) {
  const int r = a.r;
  a.hot = HOT_NONE;
  a.hot_term = 0;
  a.n_chunks = 1;
  a.rw = a.sw = a.qcap = 0;
  a.nseg = 0;
  if (r > 64 && !legacy_wide) {
    // warp-tile kernel: segments of 32*cpt candidates; cost per node quad
    // ~ nseg * (6 cpt + 12) instructions (hot loop + per-quad ballots / loop overhead)
    int best_cpt = 0, best_nseg = 0;
    double best = 1e30;
    for (int cpt : {4, 8, 12, 16, 20, 24, 32}) {
      const int64_t seg = 32 * (int64_t)cpt;
      const int64_t nseg = ((int64_t)r + seg - 1) / seg;
      if (nseg > kMaxSeg) continue;
      const double cost = (double)nseg * (6.0 * cpt + 12.0);
      if (cost < best - 1e-9) { best = cost; best_cpt = cpt; best_nseg = (int)nseg; }
    }
    if (best_cpt) {
      // (levels reading an int64 ancestor take the generic prologue: no hot filter, reading #22)
      for (int t = 0; t < a.n_terms && !a.pv64_any; t++) {
        const Term& T = a.terms[t];
        if ((T.kind == T_DIVX || T.kind == T_DIVPROD) && T.variant == V16) { a.hot = HOT_DIVX; a.hot_term = t; break; }
        if (T.kind == T_MULX && T.variant == V16) { a.hot = HOT_MULX; a.hot_term = t; break; }
      }
      // Divisor filters over ranges that already span several segments: finer segments (the
      // smallest cpt >= 8 that fits kMaxSeg) let small node values skip more candidates
      // (C5 9.44 -> 9.33 ms measured; multiples filters and single-segment levels lose, so
      // they keep the cost-model choice).  Without segment bounds (ATF_FLAG_NO_SEG_BOUNDS)
      // finer segments only add loop overhead.
      const int fine = (seg_bounds && a.hot == HOT_DIVX && best_nseg >= 2) ? 8 : 0;
      if (fine) {
        // finer segments: more node quads fall outside a segment's |x| bounds
        for (int cpt : {4, 8, 12, 16, 20, 24, 32}) {
          if (cpt < fine) continue;
          const int64_t seg = 32 * (int64_t)cpt, nseg = ((int64_t)r + seg - 1) / seg;
          if (nseg <= kMaxSeg) { best_cpt = cpt; best_nseg = (int)nseg; break; }
        }
      }
      a.kind = K_WTILE;
      a.cpt = best_cpt;
      a.nseg = best_nseg;
      a.chunk = 32 * best_cpt * best_nseg;
      // small and mid-size frontiers: fewer nodes per warp tile (power of two, >= 4 = one
      // node quad of the hot loop) until ~256 tiles per SM exist: more tiles shorten the tail
      // of heavy tiles (nodes with thousands of children); measured sweet spot on C5
      int tnodes = kWT;
      const uint64_t want_tiles = 148ull * (uint64_t)g_tiles_per_sm.load();
      while (tnodes > 4 && (a.n_parents + tnodes - 1) / tnodes < want_tiles) tnodes >>= 1;
      a.tile_nodes = tnodes;
      // 8 warps per CTA unless the level has too few tiles to give every SM a full CTA
      const uint64_t tiles = (a.n_parents + tnodes - 1) / tnodes;
      const uint64_t per_sm = (tiles + 147) / 148;
      a.block = 32 * (int)std::min<uint64_t>(8, std::max<uint64_t>(1, per_sm));
      a.smem_bytes = wtile_layout(a, words).total;
      return;
    }
  }
  if (r <= 64 && a.nf_ok && !legacy_wide) {
    a.kind = K_NFAST;
    a.block = 256;
    a.cpt = 1;
    a.tile_nodes = 32 * kNfNPL;
    a.chunk = r;
    a.smem_bytes = 0;
    return;
  }
  if (r <= 64) {
    a.kind = K_NARROW;
    a.block = 256;
    a.cpt = 1;
    a.tile_nodes = 256 * 4;  // kNarrowNPT nodes per thread
    a.chunk = r;
  } else {
    a.kind = K_WIDE;
    for (int t = 0; t < a.n_terms && !a.pv64_any; t++) {
      const Term& T = a.terms[t];
      if ((T.kind == T_DIVX || T.kind == T_DIVPROD) && T.variant == V16) { a.hot = HOT_DIVX; a.hot_term = t; break; }
      if (T.kind == T_MULX && T.variant == V16) { a.hot = HOT_MULX; a.hot_term = t; break; }
    }
    // cost per useful pair ~ (1.6 instructions + queue/loop overhead per node quad) x
    // padding waste; blocks under 256 threads lose latency hiding at the tile barriers
    double best = 1e30;
    for (int cpt : {4, 8, 16}) {
      int64_t per = ((int64_t)r + cpt - 1) / cpt;
      int B = (int)std::min<int64_t>(256, (per + 31) / 32 * 32);
      int64_t nch = ((int64_t)r + (int64_t)B * cpt - 1) / ((int64_t)B * cpt);
      double cost = (1.6 + 6.0 / (4.0 * cpt)) * (double)((int64_t)B * cpt * nch) / r;
      if (B < 256) cost *= 1.1;
      if (cost < best - 1e-9) { best = cost; a.cpt = cpt; a.block = B; a.n_chunks = nch; }
    }
    if (r >= 2048 && r <= 4096) {
      // wide ranges: 128-thread CTAs with 16-32 candidates per thread, so that 8 CTAs fit
      // an SM (64 registers, <= 26 KB shared) and cover each other's tile barriers
      a.cpt = r > 2048 ? 32 : 16;
      a.block = (int)(((int64_t)r + a.cpt * 32 - 1) / (a.cpt * 32) * 32);
      a.n_chunks = 1;
    }
    a.chunk = a.block * a.cpt;
    a.rw = a.chunk / 32;
    a.sw = (a.rw + 31) / 32;
    const int smem_budget = a.block <= 128 ? 26 * 1024 : 48 * 1024;
    // the slow-path queue holds one entry per (node quad, thread): it cannot overflow
    int nt = a.n_chunks > 1 ? 4 : std::max(4, std::min(256, ((1 << 18) / a.chunk + 3) / 4 * 4));
    for (;;) {
      a.tile_nodes = nt;
      a.qcap = nt / 4 * a.block;
      if (nt <= 4 || expand_layout(a, words).total <= smem_budget) break;
      nt -= 4;
    }
  }
  a.smem_bytes = expand_layout(a, words).total;
}

// ---------------------------------------------------------------- pinned result slots
// run_levels_async reads each group's level total through a pinned 4 KB block (an asynchronous
// copy per group instead of one synchronising copy per round).  The blocks are pooled per
// process: a fresh space (one per request) does not pay a cudaMallocHost.
constexpr size_t kPinSlotBytes = 64;  // per group: total u64 | overflow u32 | pad | tail totals u64[4]
static std::mutex g_pin_mu;
static std::vector<void*> g_pin_free;
static unsigned long long* pinned_slot_acquire() {
  {
    std::lock_guard<std::mutex> lk(g_pin_mu);
    if (!g_pin_free.empty()) {
      void* p = g_pin_free.back();
      g_pin_free.pop_back();
      return (unsigned long long*)p;
    }
  }
  void* p = nullptr;
  if (cudaMallocHost(&p, kMaxGroups * kPinSlotBytes) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return (unsigned long long*)p;
}
static void pinned_slot_release(unsigned long long* p) {
  if (!p) return;
  std::lock_guard<std::mutex> lk(g_pin_mu);
  g_pin_free.push_back(p);
}

// ---------------------------------------------------------------- device setup
static atf_status ensure_device(atf_space* s) {
  CUDA_TRY(s, cudaSetDevice(s->opts.device));
  if (s->dev_ready) return ATF_OK;
  if (!s->opts.alloc) {
    // cudaMallocAsync path: keep freed blocks in the device's default pool so that a new
    // space (e.g. one per request) does not re-map its arenas
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, s->opts.device) == cudaSuccess) {
      uint64_t keep = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    }
    cudaGetLastError();
  }
  // one device block for every parameter's tables and the small scratch words, filled by
  // one host -> device copy: per parameter [values rp][divisibility magics rp][|values| rp]
  // (rp = r rounded up to 128; the wide kernel reads 16-byte vectors of the last two on
  // chunked ranges), then [values sorted ascending r][their positions r] (encode).
  // magic(x) = ceil(2^32/|x|) mod 2^32 (0 for |x| == 1); magic(0) = 2^16, which no 16-bit
  // x != 0 has, so the wide kernel's uniform test (n * magic mod 2^32) < 2^16 never accepts
  // x == 0 for n != 0.  Padding: value 1, magic 2^16, |value| 1.
  size_t np = s->params.size();
  std::vector<size_t> off_range(np), off_sorted(np);
  size_t words = 0;
  for (size_t p = 0; p < np; p++) {
    const size_t r = s->params[p].values.size(), rp = (r + 127) / 128 * 128;
    off_range[p] = words;
    words += 3 * rp;
    off_sorted[p] = words;
    words += (2 * r + 3) / 4 * 4;
  }
  // int64 parameters: their int64 value tables (8-byte aligned), reading #22
  std::vector<size_t> off_range64(np, 0);
  for (size_t p = 0; p < np; p++)
    if (s->params[p].v64) {
      words = (words + 3) / 4 * 4;
      off_range64[p] = words;
      words += 2 * s->params[p].values64.size();
    }
  words = (words + 3) / 4 * 4;
  // totals u64[kMaxGroups] | ovf[kMaxGroups] | tile counters[kMaxGroups] | bad[4] | root[16]:
  // one memset per level round resets [totals, ovf, counters], one copy reads [totals, ovf]
  const size_t off_scr = words;
  words += 2 * kMaxGroups + kMaxGroups + kMaxGroups + 4 + 16 + 2 * kMaxGroups;  // + pairs u64 (timing)
  std::vector<int32_t> host(words, 0);
  for (size_t p = 0; p < np; p++) {
    auto& v = s->params[p].values;
    const size_t r = v.size(), rp = (r + 127) / 128 * 128;
    int32_t* buf = host.data() + off_range[p];
    for (size_t j = 0; j < rp; j++) {
      const bool real = j < r;
      const uint32_t ax = real ? (v[j] < 0 ? 0u - (uint32_t)v[j] : (uint32_t)v[j]) : 1u;
      buf[j] = real ? v[j] : 1;
      buf[rp + j] = (int32_t)(real ? (ax ? 0xffffffffu / ax + 1u : 0x10000u) : 0x10000u);
      buf[2 * rp + j] = (int32_t)ax;
    }
    std::vector<int32_t> idx(r);
    std::iota(idx.begin(), idx.end(), 0);
    std::sort(idx.begin(), idx.end(), [&](int32_t x, int32_t y) { return v[x] < v[y]; });
    int32_t* sb = host.data() + off_sorted[p];
    for (size_t j = 0; j < r; j++) {
      sb[j] = v[idx[j]];
      sb[r + j] = idx[j];
    }
  }
  for (size_t p = 0; p < np; p++)
    if (s->params[p].v64)
      std::memcpy(host.data() + off_range64[p], s->params[p].values64.data(), 8 * s->params[p].values64.size());
  s->table_bytes = words * 4;
  s->d_table = (int32_t*)dalloc(s, s->table_bytes);
  if (!s->d_table) return fail(s, ATF_ERR_OOM, "parameter tables (%zu bytes)", s->table_bytes);
  // pageable source: the call returns once `host` has been staged
  CUDA_TRY(s, cudaMemcpyAsync(s->d_table, host.data(), s->table_bytes, cudaMemcpyHostToDevice,
                              (cudaStream_t)s->opts.stream));
  s->d_range.assign(np, nullptr);
  s->d_sorted.assign(np, nullptr);
  s->d_range64.assign(np, nullptr);
  for (size_t p = 0; p < np; p++) {
    s->d_range[p] = s->d_table + off_range[p];
    s->d_sorted[p] = s->d_table + off_sorted[p];
    if (s->params[p].v64) s->d_range64[p] = reinterpret_cast<const int64_t*>(s->d_table + off_range64[p]);
  }
  int32_t* scr = s->d_table + off_scr;
  s->d_totals = (unsigned long long*)scr;
  s->d_ovf = (unsigned int*)(scr + 2 * kMaxGroups);
  s->d_counter = (unsigned int*)(scr + 3 * kMaxGroups);
  s->d_bad = (unsigned int*)(scr + 4 * kMaxGroups);
  s->d_root = (uint32_t*)(scr + 4 * kMaxGroups + 4);
  s->d_pairs = (unsigned long long*)(scr + 4 * kMaxGroups + 20);
  // level totals and flags come back with the round's synchronisation (pageable is enough):
  // host mirror of [totals u64[kMaxGroups] | ovf u32[kMaxGroups]]
  s->h_ctl.assign(3 * kMaxGroups, 0);
  s->h_totals = reinterpret_cast<unsigned long long*>(s->h_ctl.data());
  s->h_flags = s->h_ctl.data() + 2 * kMaxGroups;
  s->arena.assign(s->groups.size(), {});
  s->gb.assign(s->groups.size(), {});
  for (auto& b : s->gb) {
    CUDA_TRY(s, cudaStreamCreateWithFlags(&b.stream, cudaStreamNonBlocking));
    CUDA_TRY(s, cudaEventCreateWithFlags(&b.fork, cudaEventDisableTiming));
    CUDA_TRY(s, cudaEventCreateWithFlags(&b.join, cudaEventDisableTiming));
    CUDA_TRY(s, cudaEventCreateWithFlags(&b.done, cudaEventDisableTiming));
  }
  s->dev_ready = true;
  return ATF_OK;
}


static atf_status ensure_buf(atf_space* s, char** p, size_t* cap, size_t bytes, const char* what) {
  if (bytes <= *cap) return ATF_OK;
  if (s->capturing) return fail(s, ATF_ERR_OOM, "%s: growth during graph capture", what);
  dfree(s, *p, *cap);
  size_t c = std::max<size_t>(bytes, *cap * 2);
  *p = (char*)dalloc(s, c);
  if (!*p) { *cap = 0; return fail(s, ATF_ERR_OOM, "%s (%zu bytes)", what, c); }
  *cap = c;
  return ATF_OK;
}

// bump allocation inside group g's arena; nullptr if no chunk has room
static char* arena_alloc(atf_space* s, int g, size_t bytes) {
  bytes = (bytes + 255) & ~(size_t)255;
  for (auto& c : s->arena[g])
    if (c.size - c.used >= bytes) {
      char* p = c.p + c.used;
      c.used += bytes;
      return p;
    }
  return nullptr;
}
static atf_status arena_grow(atf_space* s, int g, size_t need) {
  size_t total = 0;
  for (auto& c : s->arena[g]) total += c.size;
  size_t sz = std::max<size_t>({need + (need >> 3) + (1 << 20), total, (size_t)64 << 20});
  Chunk c;
  c.p = (char*)dalloc(s, sz);
  if (!c.p) return fail(s, ATF_ERR_OOM, "arena chunk of %zu bytes", sz);
  c.size = sz;
  s->arena[g].push_back(c);
  return ATF_OK;
}
// largest free tail of the arena (chunk index, bytes)
static size_t arena_tail(atf_space* s, int g, int* which) {
  size_t best = 0;
  *which = -1;
  for (size_t i = 0; i < s->arena[g].size(); i++) {
    auto& c = s->arena[g][i];
    if (c.size - c.used > best) { best = c.size - c.used; *which = (int)i; }
  }
  return best;
}

static void drop_graph(atf_space* s) {
  if (s->graph_exec) cudaGraphExecDestroy(s->graph_exec);
  s->graph_exec = nullptr;
  s->replays = 0;
}

static void release_device(atf_space* s) {
  drop_graph(s);
  if (s->cap_stream) cudaStreamDestroy(s->cap_stream);
  if (s->cap_ev) cudaEventDestroy(s->cap_ev);
  s->cap_stream = nullptr;
  s->cap_ev = nullptr;
  dfree(s, (char*)s->d_dflags, 8 * (kDistMaxRounds + 2));
  s->d_dflags = nullptr;
  s->dflags_has_ipc = false;
  s->dlog = atf_space::DistLog{};
  for (auto ev : s->dist_ev) cudaEventDestroy(ev);
  s->dist_ev.clear();
  if (s->h_gate) cudaFreeHost(s->h_gate);
  s->h_gate = s->d_gate = nullptr;
  for (size_t g = 0; g < s->arena.size(); g++)
    for (auto& c : s->arena[g]) dfree(s, c.p, c.size);
  s->arena.clear();
  dfree(s, s->d_table, s->table_bytes);
  s->d_table = nullptr;
  s->table_bytes = 0;
  s->d_range.clear();
  s->d_range64.clear();
  s->d_sorted.clear();
  dfree(s, s->d_status, s->status_cap * 8);
  dfree(s, (char*)s->d_replay, s->replay_cap * 12 * kMaxGroups);
  s->d_replay = nullptr;
  s->replay_cap = 0;
  s->replay_ok = false;
  drop_graph(s);
  for (auto& b : s->gb) {
    dfree(s, b.scratch, b.scratch_cap);
    dfree(s, (char*)b.stash, b.stash_cap);
    dfree(s, b.masks, b.masks_cap);
    dfree(s, (char*)b.status, b.status_cap * 8);
    dfree(s, b.pbuf, b.pbuf_cap);
    if (b.stream) {
      cudaStreamSynchronize(b.stream);
      cudaStreamDestroy(b.stream);
    }
    if (b.fork) cudaEventDestroy(b.fork);
    if (b.join) cudaEventDestroy(b.join);
    if (b.done) cudaEventDestroy(b.done);
  }
  s->gb.clear();
  pinned_slot_release(s->h_pin);
  s->h_pin = nullptr;
  for (auto& pm : s->peers) cudaIpcCloseMemHandle(pm.base);
  s->peers.clear();
  s->d_counter = nullptr;
  s->d_totals = nullptr;
  s->d_ovf = nullptr;
  s->d_bad = nullptr;
  s->d_pairs = nullptr;
  s->d_root = nullptr;
  for (auto& ev : s->events)
    for (auto& e : ev) {
      cudaEventDestroy(e.first);
      cudaEventDestroy(e.mid);
      cudaEventDestroy(e.second);
    }
  s->events.clear();
  s->d_status = nullptr;
  s->h_totals = nullptr;
  s->h_flags = nullptr;
  s->dev_ready = false;
}

// ---------------------------------------------------------------- generation driver
// Expand level k of group g from `parents` (n_parents nodes) into the group's arena.
// Queues work only; the level total lands in d_totals[g].
struct Pending {
  int g, k;
  uint64_t n_parents;
  const uint32_t* parents;
  uint64_t* csr;
  uint32_t* child;
  uint64_t cap;
  int chunk;  // arena chunk holding the child region
  size_t child_off;
  bool joined = false;  // ran on the group's own stream (join event recorded)
  int kind = 0;         // 0 one level, 1 tail count, 2 tail emit
};

// device tables of a level: candidate values / magics / |values| and every referenced
// ancestor's value and magic table (see ensure_device: [values rp][magic rp][abs rp])
static void fill_level_ptrs(atf_space* s, const LevelPlan& lp, LevelArgs& a) {
  a.cand = s->d_range[lp.param];
  a.cand64 = s->d_range64[lp.param];  // int64 parameter: cand holds positions (reading #22)
  const size_t rp = ((size_t)lp.r + 127) / 128 * 128;
  a.cand_magic = reinterpret_cast<const uint32_t*>(s->d_range[lp.param]) + rp;
  a.cand_abs = reinterpret_cast<const uint32_t*>(s->d_range[lp.param]) + 2 * rp;
  a.r = lp.r;
  a.pv64_any = 0;
  for (int i = 0; i < a.n_pv; i++) {
    a.pv_range[i] = s->d_range[lp.pv_param[i]];
    a.pv_range64[i] = s->d_range64[lp.pv_param[i]];
    if (a.pv_range64[i]) a.pv64_any = 1;
    const size_t rpi = (s->params[lp.pv_param[i]].values.size() + 127) / 128 * 128;
    a.pv_magic[i] = reinterpret_cast<const uint32_t*>(s->d_range[lp.pv_param[i]]) + rpi;
  }
}

static atf_status queue_level(atf_space* s, int g, int k, const uint32_t* parents, uint64_t n_parents, Pending& pd,
                              bool own_stream, uint64_t known = UINT64_MAX) {
  GroupPlan& gp = s->groups[g];
  LevelPlan& lp = gp.levels[k];
  cudaStream_t st = (cudaStream_t)s->opts.stream;  // allocations, memsets
  auto& gbf = s->gb[g];                            // this group's buffers and launch stream
#ifdef ATF_HOST_PROF
  using hclk = std::chrono::steady_clock;
  const auto q0 = hclk::now();
#endif
  LevelArgs a = lp.proto;
  a.parent_rec = parents;
  a.n_parents = n_parents;
  fill_level_ptrs(s, lp, a);
  const bool seg_bounds = (s->opts.flags & ATF_FLAG_NO_SEG_BOUNDS) == 0;
  choose_geometry(a, gp.words, (s->opts.flags & ATF_FLAG_LEGACY_WIDE) != 0, seg_bounds);
  a.seg_on = (a.kind == K_WTILE && a.hot != HOT_NONE && seg_bounds) ? 1 : 0;
  if (a.kind == K_WTILE && a.hot != HOT_NONE && !seg_bounds) {
    // every pair is evaluated: bounds that no node quad can fall outside of
    for (int sg = 0; sg < kMaxSeg; sg++) { a.seg_lo[sg] = 0u; a.seg_hi[sg] = 0xffffffffu; }
  } else if (a.kind == K_WTILE && a.hot != HOT_NONE) {
    if (lp.seg_cpt != a.cpt) {  // per-segment |x| bounds of the hot filter (cached per level)
      const std::vector<int32_t>& v = s->params[lp.param].values;
      const int seg = 32 * a.cpt;
      for (int sg = 0; sg < kMaxSeg; sg++) {
        uint32_t lo = 0xffffffffu, hi = 0u;
        for (int j = sg * seg; j < std::min((int)v.size(), (sg + 1) * seg); j++) {
          const uint32_t ax = (uint32_t)(v[j] < 0 ? -(int64_t)v[j] : (int64_t)v[j]);
          if (ax == 0) { lo = 0u; hi = 0xffffffffu; break; }
          lo = std::min(lo, ax);
          hi = std::max(hi, ax);
        }
        lp.seg_lo[sg] = lo;
        lp.seg_hi[sg] = hi;
      }
      lp.seg_cpt = a.cpt;
    }
    for (int sg = 0; sg < kMaxSeg; sg++) { a.seg_lo[sg] = lp.seg_lo[sg]; a.seg_hi[sg] = lp.seg_hi[sg]; }
  }
  // warp-tile levels are written in place (deferred decoupled look-back) unless
  // ATF_FLAG_STASH_EMIT asks for the stash + scan + level_emit path
  a.pairs_out = (s->opts.flags & ATF_FLAG_TIMING) ? s->d_pairs + g : nullptr;
  // mid-width nf_ok levels: the NVRTC-specialised exact-mask kernel (jit.cpp), tiles of 32
  // nodes, stash output protocol of the warp-tile kernel
  const bool jit_ok = !(s->opts.flags & (ATF_FLAG_NO_JIT | ATF_FLAG_LEGACY_WIDE));
  void* wide_jit = nullptr;
  // (frontiers of >= 4096 nodes: lane = node needs enough warp tiles to fill the GPU; a
  // small frontier with many children per node stays on the warp-tile kernel)
  if (jit_ok && a.kind == K_WTILE && a.nf_ok && a.r <= kWideJitMax && n_parents >= 4096) {
    if (!lp.wide_jit_tried) {
      const auto& vals = s->params[lp.param].values;
      std::vector<uint32_t> mags(vals.size());
      for (size_t j = 0; j < vals.size(); j++) {
        const uint32_t ax = vals[j] < 0 ? 0u - (uint32_t)vals[j] : (uint32_t)vals[j];
        mags[j] = ax ? 0xffffffffu / ax + 1u : 0x10000u;  // as ensure_device
      }
      lp.wide_jit = jit_wide_kernel(a, gp.words, vals, mags);
      lp.wide_jit_tried = true;
    }
    wide_jit = lp.wide_jit;
    if (wide_jit) {
      a.tile_nodes = kWT;
      a.n_chunks = 1;
    }
  }
  s->data[g][k].seg_skip = a.kind == K_WTILE && a.hot != HOT_NONE && seg_bounds && !wide_jit;
  a.n_tiles = a.n_chunks > 1 ? n_parents * (uint64_t)a.n_chunks
                             : (n_parents + (uint64_t)a.tile_nodes - 1) / (uint64_t)a.tile_nodes;
  // tiny wide levels: one launch, in place (decoupled look-back over <= 16 warp tiles; with
  // more tiles the waits cost more than the two saved launches: DESIGN.md §5).  Otherwise
  // children go to per-tile stash segments and scan_kernel + level_emit_kernel place them.
  a.direct = (a.kind == K_WTILE && !wide_jit && !(s->opts.flags & ATF_FLAG_LEGACY_WIDE) &&
              a.n_tiles <= (uint64_t)g_direct_tiles.load()) ? 1 : 0;
  if (a.kind == K_WTILE) a.smem_bytes = wtile_layout(a, gp.words).total;
  if (a.smem_bytes > 227 * 1024)
    return fail(s, ATF_ERR_LIMIT, "level %d of group %d needs %d bytes of shared memory", k, g, a.smem_bytes);
  if (a.n_tiles >= 0xffffffffull) return fail(s, ATF_ERR_LIMIT, "level %d of group %d needs %llu tiles", k, g,
                                              (unsigned long long)a.n_tiles);
  atf_status e = ATF_OK;
  // CSR of the parent level (exact size), then the child region = largest free tail
  size_t csr_bytes = (n_parents + 1) * 8;
  char* csr = arena_alloc(s, g, csr_bytes);
  if (!csr) {
    if ((e = arena_grow(s, g, csr_bytes + n_parents * gp.words * 4))) return e;
    csr = arena_alloc(s, g, csr_bytes);
  }
  // child region: the largest free tail, grown up front to an estimate of the level's
  // size (the exact bound n_parents * r when small, else the previous level's branching
  // factor x 2) so that a fresh space rarely re-runs a level after an overflow
  uint64_t est;
  const uint64_t exact = n_parents * (uint64_t)lp.r;
  if (exact <= (1ull << 24)) {
    est = exact;
  } else if (k >= 2 && s->data[g][k - 2].n > 0) {
    const double bf = (double)s->data[g][k - 1].n / (double)s->data[g][k - 2].n;
    est = (uint64_t)std::min<double>((double)exact, 2.0 * bf * (double)n_parents + 1024.0);
  } else {
    est = std::min<uint64_t>(exact, 16 * n_parents + 1024);
  }
  est = std::min<uint64_t>(est, (4ull << 30) / (gp.words * 4));  // at most 4 GB up front
  if (known != UINT64_MAX) est = known;  // replay: the exact size from the previous generation
  int which = -1;
  size_t tail = arena_tail(s, g, &which);
  const size_t want = std::max<size_t>((size_t)est * gp.words * 4, (size_t)gp.words * 4 * 64);
  if (tail < want) {
    if ((e = arena_grow(s, g, want))) return e;
    tail = arena_tail(s, g, &which);
  }
  Chunk& c = s->arena[g][which];
  size_t off = (c.used + 255) & ~(size_t)255;
  uint32_t* child = (uint32_t*)(c.p + off);
  uint64_t cap = (c.size - off) / (gp.words * 4);
  if (known != UINT64_MAX) {  // replay: reserve now (no sync before the next level is queued)
    cap = known;
    c.used = off + ((known * gp.words * 4 + 255) & ~(uint64_t)255);
  }
  a.child_rec = child;
  a.child_cap = cap;
  a.csr = (uint64_t*)csr;
  a.status = s->d_status;
  a.tile_counter = s->d_counter + g;
  a.total_out = s->d_totals + g;
  a.overflow_flag = s->d_ovf + g;
  // every level: the expand kernel writes tile stash segments; scan_kernel turns the tile
  // totals into tile bases; level_emit_kernel places the segments and fixes the CSR
  uint64_t* scan_out = nullptr;
  unsigned long long* scan_status = nullptr;
  unsigned int* scan_counter = nullptr;
  uint32_t* piece_tile = nullptr;
  uint64_t piece_cap = 0;
  {
    // stash: the level's estimated size (or the exact size after an overflow), not the
    // whole arena tail
    const uint64_t stash_recs = a.direct ? 16 : std::min<uint64_t>(cap, std::max<uint64_t>({est + est / 4,
                                                                             (uint64_t)1 << 16, s->stash_hint}));
    if ((e = ensure_buf(s, (char**)&gbf.stash, &gbf.stash_cap, (size_t)stash_recs * gp.words * 4, "stash")))
      return e;
    a.stash = gbf.stash;
    a.stash_cap = gbf.stash_cap / (gp.words * 4);
    // scratch: tile_seg u64[n] | tile_base u64[n+1] | tile_total u32[n] (pad) |
    //          scan status u64[ceil(n/1024)+1] | scan counter u32 | stash_top u64 |
    //          piece_tile u32[stash_cap / 2^kPieceShift + 2]
    const size_t n = a.n_tiles, nscan = (n + 1023) / 1024 + 1;
    const size_t o_seg = 0, o_base = o_seg + 8 * n, o_tot = o_base + 8 * (n + 1);
    const size_t o_scan = (o_tot + 4 * n + 15) & ~(size_t)15, o_cnt = o_scan + 8 * nscan, o_top = o_cnt + 16;
    const size_t o_piece = o_top + 16;
    a.piece_shift = est < (1ull << 20) ? 7 : kPieceShift;
    piece_cap = (a.stash_cap >> a.piece_shift) + 2;
    if ((e = ensure_buf(s, &gbf.scratch, &gbf.scratch_cap, o_piece + 4 * piece_cap, "tile scratch"))) return e;
    char* const d_scratch = gbf.scratch;
    a.tile_seg = (unsigned long long*)(d_scratch + o_seg);
    scan_out = (uint64_t*)(d_scratch + o_base);
    a.tile_base = scan_out;
    a.tile_total = (uint32_t*)(d_scratch + o_tot);
    scan_status = (unsigned long long*)(d_scratch + o_scan);
    scan_counter = (unsigned int*)(d_scratch + o_cnt);
    a.stash_top = (unsigned long long*)(d_scratch + o_top);
    piece_tile = (uint32_t*)(d_scratch + o_piece);
    a.piece_tile = piece_tile;
    CUDA_TRY(s, cudaMemsetAsync(d_scratch + o_scan, 0, o_top + 16 - o_scan, st));
  }
#ifdef ATF_HOST_PROF
  const auto q1 = hclk::now();
#endif
  if (a.direct) {
    const size_t need = (size_t)a.n_tiles + 1;
    if (need > gbf.status_cap) {
      dfree(s, (char*)gbf.status, gbf.status_cap * 8);
      gbf.status_cap = std::max<size_t>(need, 64);
      gbf.status = (unsigned long long*)dalloc(s, gbf.status_cap * 8);
      if (!gbf.status) { gbf.status_cap = 0; return fail(s, ATF_ERR_OOM, "tile status"); }
    }
    a.status = gbf.status;
    CUDA_TRY(s, cudaMemsetAsync(gbf.status, 0, need * 8, st));
  }
  // narrow fast levels: pass 1 writes per-parent accept masks, pass 2 the children in place
  if (a.kind == K_NFAST) {
    a.mask_bytes = a.r <= 8 ? 1 : (a.r <= 16 ? 2 : (a.r <= 32 ? 4 : 8));
    if ((e = ensure_buf(s, &gbf.masks, &gbf.masks_cap, (size_t)n_parents * a.mask_bytes + 16, "accept masks")))
      return e;
    a.masks = gbf.masks;
  }
  // (tile counter, overflow flag and total of the group were reset by run_levels' round memset)
  // the level's kernels run on the group's stream after the allocations / memsets above;
  // run_levels joins the group streams back into the space's stream
  const bool serial = !own_stream || (s->opts.flags & ATF_FLAG_SERIAL_GROUPS) != 0;
  cudaStream_t ls = serial ? st : gbf.stream;
  if (!serial) {
    CUDA_TRY(s, cudaEventRecord(gbf.fork, st));
    CUDA_TRY(s, cudaStreamWaitEvent(gbf.stream, gbf.fork, 0));
  }
  bool timing = (s->opts.flags & ATF_FLAG_TIMING) != 0;
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k].first, ls));
  if (a.kind == K_NFAST && !lp.jit_tried && !(s->opts.flags & (ATF_FLAG_NO_JIT | ATF_FLAG_LEGACY_WIDE))) {
    const auto& vals = s->params[lp.param].values;
    std::vector<uint32_t> mags(vals.size());
    for (size_t j = 0; j < vals.size(); j++) {
      const uint32_t ax = vals[j] < 0 ? 0u - (uint32_t)vals[j] : (uint32_t)vals[j];
      mags[j] = ax ? 0xffffffffu / ax + 1u : 0x10000u;  // ceil(2^32/|x|) mod 2^32 (see ensure_device)
    }
    lp.jit = jit_nfast_kernel(a, gp.words, vals, mags);
    lp.jit_tried = true;
  }
  const bool use_jit = a.kind == K_NFAST && lp.jit && !(s->opts.flags & (ATF_FLAG_NO_JIT | ATF_FLAG_LEGACY_WIDE));
  int ce = wide_jit ? jit_wide_launch(wide_jit, a, gp.words, ls)
                    : (use_jit ? jit_nfast_launch(lp.jit, a, ls) : launch_expand(a, gp.words, ls));
  LevelData& ld = s->data[g][k];
  ld.cpt = a.kind == K_WTILE && !wide_jit ? a.cpt : 0;
  ld.nseg = a.kind == K_WTILE && !wide_jit ? a.nseg : 0;
  ld.launches += a.direct ? 1 : 3;
  if (ce) return fail(s, ATF_ERR_CUDA, "expand launch (group %d level %d): %s", g, k, cudaGetErrorString((cudaError_t)ce));
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k].mid, ls));
  s->data[g][k].kernel = wide_jit ? 7 : (use_jit ? 4 : a.kind);
  if (a.direct) {
    // nothing more: the expand kernel placed the level
  } else if (a.kind == K_NFAST) {
    ce = launch_scan_u32(a.tile_total, scan_out, (int64_t)a.n_tiles, scan_status, scan_counter, ls);
    if (!ce) ce = launch_nfast_emit(a, gp.words, ls);
    if (ce) return fail(s, ATF_ERR_CUDA, "level scan/emit (group %d level %d): %s", g, k, cudaGetErrorString((cudaError_t)ce));
  } else {
    ce = launch_scan_u32(a.tile_total, scan_out, (int64_t)a.n_tiles, scan_status, scan_counter, ls, piece_tile, piece_cap,
                         a.piece_shift);
    if (!ce) ce = launch_level_emit(a, gp.words, ls);
    if (ce) return fail(s, ATF_ERR_CUDA, "level scan/emit (group %d level %d): %s", g, k, cudaGetErrorString((cudaError_t)ce));
  }
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k].second, ls));
  if (!serial) CUDA_TRY(s, cudaEventRecord(gbf.join, ls));
#ifdef ATF_HOST_PROF
  {
    auto us = [](hclk::time_point x, hclk::time_point y) { return std::chrono::duration<double, std::micro>(y - x).count(); };
    const auto q2 = hclk::now();
    fprintf(stderr, "[atf host]   g%d k%d: setup+alloc %.1f us, launch %.1f us\n", g, k, us(q0, q1), us(q1, q2));
  }
#endif
  pd.joined = !serial;
  pd = Pending{g, k, n_parents, parents, (uint64_t*)csr, child, cap, which, off, pd.joined};
  return ATF_OK;
}

// ---------------------------------------------------------------- fused narrow tail
// Candidate tables and ancestor levels of a tail's levels (the NVRTC generator's inputs).
static void tail_jit_inputs(const atf_space* s, const GroupPlan& gp, int k0, int nl,
                            std::vector<std::vector<int32_t>>& cx, std::vector<std::vector<uint32_t>>& cm,
                            std::vector<std::vector<int>>& pv_level) {
  cx.assign(nl, {});
  cm.assign(nl, {});
  pv_level.assign(nl, {});
  for (int d = 0; d < nl; d++) {
    const LevelPlan& lp = gp.levels[k0 + d];
    cx[d] = s->params[lp.param].values;
    for (int32_t v : cx[d]) {
      const uint32_t ax = v < 0 ? 0u - (uint32_t)v : (uint32_t)v;
      cm[d].push_back(ax ? 0xffffffffu / ax + 1u : 0x10000u);  // as ensure_device
    }
    for (int q : lp.pv_param)
      pv_level[d].push_back((int)(std::find(gp.members.begin(), gp.members.end(), q) - gp.members.begin()));
  }
}

// The generator's view of a tail starting at k0 (level prototypes; no device pointers).
static TailArgs tail_protos(const GroupPlan& gp, int k0) {
  TailArgs t;
  std::memset(&t, 0, sizeof t);
  t.nl = (int)gp.levels.size() - k0;
  for (int d = 0; d < t.nl; d++) {
    t.lv[d] = gp.levels[k0 + d].proto;
    t.lv[d].r = gp.levels[k0 + d].r;
  }
  return t;
}

// First level of group g's fused narrow tail for the generic tail kernels (expand.cuh): the
// longest run of trailing levels (2..kMaxTail) that are all narrow fast levels with
// 1 <= r <= 32 and whose per-warp emit buffers (32 * r * words * 4 bytes per level) fit 16 KB;
// -1 if none.
static int tail_start_generic(const atf_space* s, int g) {
  if (s->opts.flags & (ATF_FLAG_NO_TAIL | ATF_FLAG_LEGACY_WIDE | ATF_FLAG_GENERIC_ONLY)) return -1;
  const GroupPlan& gp = s->groups[g];
  const int L = (int)gp.levels.size();
  int k0 = L, bytes = 0;
  while (k0 > 0 && L - k0 < kMaxTail) {
    const LevelPlan& lp = gp.levels[k0 - 1];
    if (!lp.proto.nf_ok || lp.generic || lp.r < 1 || lp.r > 32) break;
    const int b = 32 * lp.r * gp.words * 4;
    if (bytes + b > 16 * 1024) break;
    bytes += b;
    k0--;
  }
  return L - k0 >= 2 ? k0 : -1;
}

// The NVRTC tail has neither limit for its inner levels: it takes r <= 64 (u64 masks) above
// the leaf level and stages any subtree size in parts.  Its longer run (-1 if it is not longer
// than the generic one, or NVRTC is off).
static int tail_start_ext(const atf_space* s, int g) {
  if (s->opts.flags & (ATF_FLAG_NO_TAIL | ATF_FLAG_LEGACY_WIDE | ATF_FLAG_GENERIC_ONLY | ATF_FLAG_NO_JIT)) return -1;
  const GroupPlan& gp = s->groups[g];
  const int L = (int)gp.levels.size();
  int ke = L;
  while (ke > 0 && L - ke < kMaxTail) {
    const LevelPlan& lp = gp.levels[ke - 1];
    if (!lp.proto.nf_ok || lp.generic || lp.r < 1 || lp.r > (ke == L ? 32 : 64)) break;
    ke--;
  }
  const int kc = tail_start_generic(s, g);
  return (L - ke >= 2 && (kc < 0 || ke < kc)) ? ke : -1;
}

// The tail's kernels for a start it was not built for yet (once per group and start).
static bool tail_ext_compiled(atf_space* s, int g, int ke) {
  GroupPlan& gp = s->groups[g];
  if (gp.tail_ext_k0 != ke) {
    gp.tail_ext_k0 = ke;
    std::vector<std::vector<int32_t>> cx;
    std::vector<std::vector<uint32_t>> cm;
    std::vector<std::vector<int>> pvl;
    tail_jit_inputs(s, gp, ke, (int)gp.levels.size() - ke, cx, cm, pvl);
    const TailArgs t = tail_protos(gp, ke);
    void* kern = jit_tail_kernels(t, gp.words, cx, cm, ke, pvl);
    gp.tail_ext_ok = kern != nullptr;
    if (kern) {
      gp.tail_jit = kern;
      gp.tail_jit_k0 = ke;
    }
  }
  return gp.tail_ext_ok;
}

// Does group g's fused tail start at level k (frontier = the level above, `frontier` nodes in
// the whole space)?  The longer NVRTC run when it compiles and its frontier holds at least
// kTailExtMinFrontier nodes (a deeper tail over a small frontier leaves most SMs idle; the
// frontier size is known when level k is reached, so the choice is made then, the same way in
// every generation and on every rank), else the generic run.
constexpr uint64_t kTailExtMinFrontier = 65536;
static bool tail_here(atf_space* s, int g, int k, uint64_t frontier) {
  const int ke = tail_start_ext(s, g);
  if (ke >= 0 && k == ke && frontier >= kTailExtMinFrontier && tail_ext_compiled(s, g, ke)) return true;
  return k == tail_start_generic(s, g);
}

// The longest tail (source tests): the NVRTC run when there is one.
static int tail_start(const atf_space* s, int g) {
  const int ke = tail_start_ext(s, g);
  return ke >= 0 ? ke : tail_start_generic(s, g);
}

// Count round of the tail of group g from frontier `parents` (level k0 - 1, n_parents nodes):
// tail_count, then one exclusive scan of the warp-tile counts per tail level.
static atf_status queue_tail_count(atf_space* s, int g, int k0, const uint32_t* parents, uint64_t n_parents,
                                   Pending& pd, bool own_stream) {
  GroupPlan& gp = s->groups[g];
  auto& T = s->tails[g];
  auto& gbf = s->gb[g];
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  const int nl = (int)gp.levels.size() - k0;
  T.k0 = k0;
  T.nl = nl;
  T.phase = 0;
  TailArgs& t = T.t;
  std::memset(&t, 0, sizeof t);
  t.nl = nl;
  t.parent_rec = parents;
  t.n_parents = n_parents;
  t.n_tiles = (n_parents + 31) / 32;
  for (int d = 0; d < nl; d++) {
    t.lv[d] = gp.levels[k0 + d].proto;
    fill_level_ptrs(s, gp.levels[k0 + d], t.lv[d]);
  }
  // scratch: tile_total u32[nl][n] | tile_base u64[nl][n+1] | scan status u64[nl][ns] | counters u32[nl]
  const size_t n = t.n_tiles, ns = (n + 1023) / 1024 + 1;
  const size_t o_tot = 0, o_base = (o_tot + 4 * nl * n + 15) & ~(size_t)15, o_stat = o_base + 8 * nl * (n + 1);
  const size_t o_cnt = o_stat + 8 * nl * ns, o_nc = (o_cnt + 4 * nl + 16 + 15) & ~(size_t)15;
  const size_t bytes = o_nc + 4 * (size_t)nl * n_parents + 16;
  atf_status e = ensure_buf(s, &gbf.scratch, &gbf.scratch_cap, bytes, "tail scratch");
  if (e) return e;
  t.tile_total = (uint32_t*)(gbf.scratch + o_tot);
  t.tile_base = (const uint64_t*)(gbf.scratch + o_base);
  t.node_cnt = (uint32_t*)(gbf.scratch + o_nc);
  CUDA_TRY(s, cudaMemsetAsync(gbf.scratch + o_stat, 0, o_nc - o_stat, st));
  const bool serial = !own_stream || (s->opts.flags & ATF_FLAG_SERIAL_GROUPS) != 0;
  cudaStream_t ls = serial ? st : gbf.stream;
  if (!serial) {
    CUDA_TRY(s, cudaEventRecord(gbf.fork, st));
    CUDA_TRY(s, cudaStreamWaitEvent(gbf.stream, gbf.fork, 0));
  }
  const bool timing = (s->opts.flags & ATF_FLAG_TIMING) != 0;
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k0].first, ls));
  if (gp.tail_jit_k0 != k0 && !(s->opts.flags & ATF_FLAG_NO_JIT)) {
    std::vector<std::vector<int32_t>> cx;
    std::vector<std::vector<uint32_t>> cm;
    std::vector<std::vector<int>> pvl;
    tail_jit_inputs(s, gp, k0, nl, cx, cm, pvl);
    gp.tail_jit = jit_tail_kernels(t, gp.words, cx, cm, k0, pvl);
    gp.tail_jit_k0 = k0;
  }
  void* tj = (s->opts.flags & ATF_FLAG_NO_JIT) ? nullptr : gp.tail_jit;
  int ce = tj ? jit_tail_launch(tj, t, false, ls) : launch_tail_count(t, gp.words, ls);
  if (ce) return fail(s, ATF_ERR_CUDA, "tail count launch (group %d): %s", g, cudaGetErrorString((cudaError_t)ce));
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k0].mid, ls));
  if (!ce)  // one launch scans every tail level's tile counts
    ce = launch_scan_u32_batch(t.tile_total, (uint64_t*)t.tile_base, (int64_t)n, nl,
                               (unsigned long long*)(gbf.scratch + o_stat), ns, (unsigned int*)(gbf.scratch + o_cnt), ls);
  if (ce) return fail(s, ATF_ERR_CUDA, "tail scan (group %d): %s", g, cudaGetErrorString((cudaError_t)ce));
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k0].second, ls));
  if (!serial) CUDA_TRY(s, cudaEventRecord(gbf.join, ls));
  s->data[g][k0].launches += 2;
  pd = Pending{};
  pd.g = g;
  pd.k = k0;
  pd.n_parents = n_parents;
  pd.parents = parents;
  pd.joined = !serial;
  pd.kind = 1;
  return ATF_OK;
}

static char* arena_take(atf_space* s, int g, size_t bytes, atf_status* e) {
  char* p = arena_alloc(s, g, bytes);
  if (!p) {
    if ((*e = arena_grow(s, g, bytes))) return nullptr;
    p = arena_alloc(s, g, bytes);
  }
  return p;
}

// Emit round of group g's tail (level sizes known from the count round): exact allocations,
// then tail_emit writes every tail level's records and the CSR of the levels above them.
static atf_status queue_tail_emit(atf_space* s, int g, Pending& pd, bool own_stream) {
  GroupPlan& gp = s->groups[g];
  auto& T = s->tails[g];
  auto& gbf = s->gb[g];
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  TailArgs& t = T.t;
  const int nl = T.nl, k0 = T.k0;
  atf_status e = ATF_OK;
  // CSR of the frontier level (its size + 1), then per tail level its records and (but the
  // last) its CSR
  t.csr[0] = (uint64_t*)arena_take(s, g, (t.n_parents + 1) * 8, &e);
  if (!t.csr[0]) return e ? e : fail(s, ATF_ERR_OOM, "tail CSR");
  for (int d = 0; d < nl; d++) {
    t.rec[d] = (uint32_t*)arena_take(s, g, std::max<uint64_t>(T.tot[d], 1) * gp.words * 4, &e);
    if (!t.rec[d]) return e ? e : fail(s, ATF_ERR_OOM, "tail records");
    if (d + 1 < nl) {
      t.csr[d + 1] = (uint64_t*)arena_take(s, g, (T.tot[d] + 1) * 8, &e);
      if (!t.csr[d + 1]) return e ? e : fail(s, ATF_ERR_OOM, "tail CSR");
    }
  }
  int off = 0;
  for (int d = 0; d < nl; d++) {
    t.buf_off[d] = off;
    off += (32 * t.lv[d].r * gp.words * 4 + 15) & ~15;
  }
  t.warp_bytes = off;
  const bool serial = !own_stream || (s->opts.flags & ATF_FLAG_SERIAL_GROUPS) != 0;
  cudaStream_t ls = serial ? st : gbf.stream;
  if (!serial) {
    CUDA_TRY(s, cudaEventRecord(gbf.fork, st));
    CUDA_TRY(s, cudaStreamWaitEvent(gbf.stream, gbf.fork, 0));
  }
  const bool timing = (s->opts.flags & ATF_FLAG_TIMING) != 0;
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k0 + 1].first, ls));
  void* tj = (s->opts.flags & ATF_FLAG_NO_JIT) ? nullptr : gp.tail_jit;
  int ce = tj ? jit_tail_launch(tj, t, true, ls) : launch_tail_emit(t, gp.words, ls);
  if (ce) return fail(s, ATF_ERR_CUDA, "tail emit launch (group %d): %s", g, cudaGetErrorString((cudaError_t)ce));
  if (timing) CUDA_TRY(s, cudaEventRecord(s->events[g][k0 + 1].second, ls));
  if (!serial) CUDA_TRY(s, cudaEventRecord(gbf.join, ls));
  s->data[g][k0].launches += 1;
  pd = Pending{};
  pd.g = g;
  pd.k = k0;
  pd.n_parents = t.n_parents;
  pd.parents = t.parent_rec;
  pd.joined = !serial;
  pd.kind = 2;
  return ATF_OK;
}

// After the emit round: the tail levels become the group's level data.
static void finish_tail(atf_space* s, int g) {
  auto& T = s->tails[g];
  const TailArgs& t = T.t;
  GroupPlan& gp = s->groups[g];
  const bool timing = (s->opts.flags & ATF_FLAG_TIMING) != 0;
  float ms_count = 0.f, ms_count_k = 0.f, ms_emit = 0.f;
  if (timing) {
    cudaEventElapsedTime(&ms_count, s->events[g][T.k0].first, s->events[g][T.k0].second);
    cudaEventElapsedTime(&ms_count_k, s->events[g][T.k0].first, s->events[g][T.k0].mid);
    cudaEventElapsedTime(&ms_emit, s->events[g][T.k0 + 1].first, s->events[g][T.k0 + 1].second);
  }
  if (T.k0 > 0) s->data[g][T.k0 - 1].csr = t.csr[0];
  for (int d = 0; d < T.nl; d++) {
    LevelData& ld = s->data[g][T.k0 + d];
    const uint64_t above = d == 0 ? t.n_parents : T.tot[d - 1];
    ld.rec = T.tot[d] ? t.rec[d] : nullptr;
    ld.n = T.tot[d];
    ld.evals = above * (uint64_t)gp.levels[T.k0 + d].r;
    ld.kernel = ((s->opts.flags & ATF_FLAG_NO_JIT) || !gp.tail_jit) ? 5 : 6;
    ld.cpt = ld.nseg = 0;
    if (d + 1 < T.nl) ld.csr = t.csr[d + 1];
    if (timing) {  // the whole tail is attributed to its first level
      ld.ms = d == 0 ? ms_count + ms_emit : 0.f;
      ld.expand_ms = d == 0 ? ms_count_k + ms_emit : 0.f;
      // product-structured tail: a level's mask is a function of the frontier node and is
      // evaluated once per frontier node (r_d pairs), not once per level-(d-1) node
      const bool prod = !(s->opts.flags & ATF_FLAG_NO_JIT) && gp.tail_jit && jit_tail_product(gp.tail_jit);
      ld.pairs = (prod && d > 0) ? t.n_parents * (uint64_t)gp.levels[T.k0 + d].r : ld.evals;
    }
  }
  T.phase = 2;
}

// Generate groups' levels [k_from, L) starting from the given frontiers; syncs once per round.
static atf_status run_levels(atf_space* s, std::vector<int> gs, std::vector<int> k_from,
                             std::vector<const uint32_t*> frontier, std::vector<uint64_t> fsize) {
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  std::vector<int> k = k_from;
#ifdef ATF_HOST_PROF  // host phases of the level-by-level rounds (diagnostic builds only)
  using hclk = std::chrono::steady_clock;
  auto hus = [](hclk::time_point a, hclk::time_point b) { return std::chrono::duration<double, std::micro>(b - a).count(); };
#endif
  for (int round = 0;; round++) {
#ifdef ATF_HOST_PROF
    const auto hp0 = hclk::now();
#endif
    char rname[48];
    snprintf(rname, sizeof rname, "atf level round %d", round);
    NvtxRange nvtx_round(rname);
    std::vector<Pending> pend;
    // levels launched this round: more than one -> one stream per group (concurrent)
    int active = 0;
    for (size_t i = 0; i < gs.size(); i++)
      if (k[i] < (int)s->groups[gs[i]].levels.size() && fsize[i] > 0 && s->groups[gs[i]].levels[k[i]].r > 0) active++;
    // one memset resets every group's level total, overflow flag and tile counter
    if (active) CUDA_TRY(s, cudaMemsetAsync(s->d_totals, 0, 16 * kMaxGroups, st));
    if (active && (s->opts.flags & ATF_FLAG_TIMING)) CUDA_TRY(s, cudaMemsetAsync(s->d_pairs, 0, 8 * kMaxGroups, st));
    for (size_t i = 0; i < gs.size(); i++) {
      int g = gs[i];
      int L = (int)s->groups[g].levels.size();
      if (k[i] >= L) continue;
      if (fsize[i] == 0 || s->groups[g].levels[k[i]].r == 0) {
        // empty frontier or empty range: every deeper level is empty
        for (int kk = k[i]; kk < L; kk++) {
          LevelData& d = s->data[g][kk];
          d.rec = nullptr;
          d.n = 0;
          d.evals = (kk == k[i]) ? fsize[i] * (uint64_t)s->groups[g].levels[kk].r : 0;
          if (kk > 0 && kk == k[i] && fsize[i] > 0) {
            // parents get an all-zero CSR
            char* csr = arena_alloc(s, g, (fsize[i] + 1) * 8);
            if (!csr) {
              atf_status e = arena_grow(s, g, (fsize[i] + 1) * 8);
              if (e) return e;
              csr = arena_alloc(s, g, (fsize[i] + 1) * 8);
            }
            CUDA_TRY(s, cudaMemsetAsync(csr, 0, (fsize[i] + 1) * 8, st));
            s->data[g][kk - 1].csr = (uint64_t*)csr;
          }
        }
        k[i] = L;
        continue;
      }
      Pending pd;
      atf_status e;
      if (s->tails[g].phase == 1) {
        e = queue_tail_emit(s, g, pd, active > 1);
      } else if (tail_here(s, g, k[i], fsize[i])) {
        e = queue_tail_count(s, g, k[i], frontier[i], fsize[i], pd, active > 1);
      } else {
        e = queue_level(s, g, k[i], frontier[i], fsize[i], pd, active > 1);
      }
      if (e) return e;
      pend.push_back(pd);
    }
    if (pend.empty()) break;
#ifdef ATF_HOST_PROF
    const auto hpq = hclk::now();
#endif
    for (auto& pd : pend)
      if (pd.joined) CUDA_TRY(s, cudaStreamWaitEvent(st, s->gb[pd.g].join, 0));  // join the group streams
    // one copy brings back [totals | overflow flags] of every group
    CUDA_TRY(s, cudaMemcpyAsync(s->h_ctl.data(), s->d_totals, 12 * kMaxGroups, cudaMemcpyDeviceToHost, st));
    for (auto& pd : pend)
      if (pd.kind == 1) {  // tail level sizes = the scans' totals
        auto& T = s->tails[pd.g];
        for (int d = 0; d < T.nl; d++)
          CUDA_TRY(s, cudaMemcpyAsync(&T.tot[d], T.t.tile_base + d * (T.t.n_tiles + 1) + T.t.n_tiles, 8,
                                      cudaMemcpyDeviceToHost, st));
      }
    CUDA_TRY(s, cudaStreamSynchronize(st));
#ifdef ATF_HOST_PROF
    fprintf(stderr, "[atf host] round %d: %zu levels, host queue %.1f us, copy+sync %.1f us\n", round, pend.size(),
            hus(hp0, hpq), hus(hpq, hclk::now()));
#endif
    unsigned long long h_pairs[kMaxGroups] = {};
    if (s->opts.flags & ATF_FLAG_TIMING)
      CUDA_TRY(s, cudaMemcpy(h_pairs, s->d_pairs, sizeof(h_pairs), cudaMemcpyDeviceToHost));
    for (auto& pd : pend) {
      size_t i = std::find(gs.begin(), gs.end(), pd.g) - gs.begin();
      if (pd.kind == 1) {
        s->tails[pd.g].phase = 1;
        continue;
      }
      if (pd.kind == 2) {
        finish_tail(s, pd.g);
        k[i] = (int)s->groups[pd.g].levels.size();
        continue;
      }
      uint64_t total = s->h_totals[pd.g];
      GroupPlan& gp = s->groups[pd.g];
      if (s->h_flags[pd.g] || total > pd.cap) {
        // child region or stash too small: grow and redo this level next round
        s->stash_hint = std::max<uint64_t>(s->stash_hint, total);
        atf_status e = arena_grow(s, pd.g, total * gp.words * 4 + (pd.n_parents + 1) * 8);
        if (e) return e;
        continue;
      }
      Chunk& c = s->arena[pd.g][pd.chunk];
      c.used = pd.child_off + ((total * gp.words * 4 + 255) & ~(uint64_t)255);
      LevelData& d = s->data[pd.g][pd.k];
      d.rec = pd.child;
      d.n = total;
      d.evals = pd.n_parents * (uint64_t)gp.levels[pd.k].r;
      if (pd.k > 0) s->data[pd.g][pd.k - 1].csr = pd.csr;
      if (s->opts.flags & ATF_FLAG_TIMING)
      {
        cudaEventElapsedTime(&d.ms, s->events[pd.g][pd.k].first, s->events[pd.g][pd.k].second);
        cudaEventElapsedTime(&d.expand_ms, s->events[pd.g][pd.k].first, s->events[pd.g][pd.k].mid);
        d.pairs = d.seg_skip ? h_pairs[pd.g] : d.evals;
      }
      frontier[i] = pd.child;
      fsize[i] = total;
      k[i]++;
    }
  }
  return ATF_OK;
}

// Level-by-level generation of every group with NO round barrier between the groups (a fresh
// space: level sizes unknown).  Each group advances on its own stream: its level's total and
// overflow flag come back through an asynchronous copy into a pinned slot, an event marks the
// group done, and the host queues that group's next level as soon as it is -- while the other
// groups' kernels keep the GPU busy, instead of every group waiting for the slowest one and the
// GPU idling while the host queues the next round (~60 us of host work per level).  Same kernels,
// same allocations and the same level data as run_levels.  Not used with ATF_FLAG_TIMING (per-round
// statistics) or ATF_FLAG_SERIAL_GROUPS.
static atf_status run_levels_async(atf_space* s) {
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  const int G = (int)s->groups.size();
  if (!s->h_pin && !(s->h_pin = pinned_slot_acquire())) return fail(s, ATF_ERR_OOM, "pinned result slots");
  std::vector<int> k(G, 0);
  std::vector<const uint32_t*> frontier(G, s->d_root);
  std::vector<uint64_t> fsize(G, 1);
  std::vector<char> busy(G, 0), finished(G, 0);
  std::vector<Pending> pend(G);
  auto slot = [&](int g) { return s->h_pin + (size_t)g * (kPinSlotBytes / 8); };
  // queue group g's next level (or finish it); returns with busy[g] set when work is in flight
  auto queue = [&](int g) -> atf_status {
    const int L = (int)s->groups[g].levels.size();
    if (k[g] >= L) { finished[g] = 1; return ATF_OK; }
    if (fsize[g] == 0 || s->groups[g].levels[k[g]].r == 0) {
      // empty frontier or empty range: every deeper level is empty
      for (int kk = k[g]; kk < L; kk++) {
        LevelData& d = s->data[g][kk];
        d.rec = nullptr;
        d.n = 0;
        d.evals = (kk == k[g]) ? fsize[g] * (uint64_t)s->groups[g].levels[kk].r : 0;
        if (kk > 0 && kk == k[g] && fsize[g] > 0) {
          atf_status e = ATF_OK;
          char* csr = arena_take(s, g, (fsize[g] + 1) * 8, &e);
          if (!csr) return e ? e : fail(s, ATF_ERR_OOM, "CSR");
          CUDA_TRY(s, cudaMemsetAsync(csr, 0, (fsize[g] + 1) * 8, st));
          s->data[g][kk - 1].csr = (uint64_t*)csr;
        }
      }
      k[g] = L;
      finished[g] = 1;
      return ATF_OK;
    }
    // this group's level total, overflow flag and tile counter (the kernels fork from st)
    CUDA_TRY(s, cudaMemsetAsync(s->d_totals + g, 0, 8, st));
    CUDA_TRY(s, cudaMemsetAsync(s->d_ovf + g, 0, 4, st));
    CUDA_TRY(s, cudaMemsetAsync(s->d_counter + g, 0, 4, st));
    Pending& pd = pend[g];
    atf_status e;
    if (s->tails[g].phase == 1) e = queue_tail_emit(s, g, pd, true);
    else if (tail_here(s, g, k[g], fsize[g])) e = queue_tail_count(s, g, k[g], frontier[g], fsize[g], pd, true);
    else e = queue_level(s, g, k[g], frontier[g], fsize[g], pd, true);
    if (e) return e;
    cudaStream_t ls = s->gb[g].stream;
    unsigned long long* h = slot(g);
    CUDA_TRY(s, cudaMemcpyAsync(h, s->d_totals + g, 8, cudaMemcpyDeviceToHost, ls));
    CUDA_TRY(s, cudaMemcpyAsync(h + 1, s->d_ovf + g, 4, cudaMemcpyDeviceToHost, ls));
    if (pd.kind == 1) {
      auto& T = s->tails[g];
      for (int d = 0; d < T.nl; d++)
        CUDA_TRY(s, cudaMemcpyAsync(h + 2 + d, T.t.tile_base + d * (T.t.n_tiles + 1) + T.t.n_tiles, 8,
                                    cudaMemcpyDeviceToHost, ls));
    }
    CUDA_TRY(s, cudaEventRecord(s->gb[g].done, ls));
    busy[g] = 1;
    return ATF_OK;
  };
  // a finished level of group g: the bookkeeping of run_levels
  auto complete = [&](int g) -> atf_status {
    busy[g] = 0;
    Pending& pd = pend[g];
    const unsigned long long* h = slot(g);
    if (pd.kind == 1) {
      auto& T = s->tails[g];
      for (int d = 0; d < T.nl; d++) T.tot[d] = h[2 + d];
      T.phase = 1;
      return ATF_OK;
    }
    if (pd.kind == 2) {
      finish_tail(s, g);
      k[g] = (int)s->groups[g].levels.size();
      return ATF_OK;
    }
    const uint64_t total = h[0];
    const uint32_t ovf = (uint32_t)(h[1] & 0xffffffffu);
    GroupPlan& gp = s->groups[g];
    if (ovf || total > pd.cap) {  // child region or stash too small: grow and redo the level
      s->stash_hint = std::max<uint64_t>(s->stash_hint, total);
      return arena_grow(s, g, total * gp.words * 4 + (pd.n_parents + 1) * 8);
    }
    Chunk& c = s->arena[g][pd.chunk];
    c.used = pd.child_off + ((total * gp.words * 4 + 255) & ~(uint64_t)255);
    LevelData& d = s->data[g][pd.k];
    d.rec = pd.child;
    d.n = total;
    d.evals = pd.n_parents * (uint64_t)gp.levels[pd.k].r;
    if (pd.k > 0) s->data[g][pd.k - 1].csr = pd.csr;
    frontier[g] = pd.child;
    fsize[g] = total;
    k[g]++;
    return ATF_OK;
  };
  atf_status e = ATF_OK;
  for (int g = 0; g < G && !e; g++) e = queue(g);
  while (!e) {
    int inflight = 0;
    for (int g = 0; g < G; g++) inflight += busy[g];
    if (!inflight) break;
    bool progressed = false;
    for (int g = 0; g < G && !e; g++) {
      if (!busy[g]) continue;
      const cudaError_t q = cudaEventQuery(s->gb[g].done);
      if (q == cudaErrorNotReady) continue;
      if (q != cudaSuccess) {
        e = fail(s, ATF_ERR_CUDA, "group %d level %d: %s", g, k[g], cudaGetErrorString(q));
        break;
      }
      progressed = true;
      if ((e = complete(g))) break;
      e = queue(g);
    }
    if (!progressed && !e) std::this_thread::yield();
  }
  // every group's work precedes what the caller queues on the space's stream next
  for (int g = 0; g < G; g++)
    if (s->gb[g].done) cudaStreamWaitEvent(st, s->gb[g].done, 0);
  if (e) {
    for (int g = 0; g < G; g++)
      if (s->gb[g].stream) cudaStreamSynchronize(s->gb[g].stream);
    return e;
  }
  return ATF_OK;
}

// ---------------------------------------------------------------- replay
// Steady-state generation of a space generated before (the bench's timed steps, a service
// regenerating the same spec): every level's size is the previous generation's, so allocations
// and launch geometry are exact up front and all level rounds are queued without a host sync
// (the per-round totals are copied into a device log); one synchronisation at the end, then
// every level's total and overflow flag is checked against the expected values.  The device
// still evaluates every pair and writes every record.  Returns ATF_ERR_STATE on any mismatch
// (the caller then regenerates level by level).
// Queue every round of a replay (no synchronisation); host-side level data as the kernels will
// leave it.  `rounds`, `expect`, `tails_done` describe the checks.
static atf_status replay_queue(atf_space* s, int& rounds_out, std::vector<ReplayExpect>& expect,
                               std::vector<std::pair<int, int>>& timed, std::vector<int>& tails_done) {
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  const size_t G = s->groups.size();
  std::vector<int> k(G, 0);
  std::vector<const uint32_t*> frontier(G, s->d_root);
  std::vector<uint64_t> fsize(G, 1);
  int round = 0;
  for (;; round++) {
    int active = 0;
    for (size_t g = 0; g < G; g++)
      if (k[g] < (int)s->groups[g].levels.size() && fsize[g] > 0 && s->groups[g].levels[k[g]].r > 0) active++;
    bool any = false;
    std::vector<Pending> pend;
    if (active) CUDA_TRY(s, cudaMemsetAsync(s->d_totals, 0, 16 * kMaxGroups, st));
    if (active && (s->opts.flags & ATF_FLAG_TIMING)) CUDA_TRY(s, cudaMemsetAsync(s->d_pairs, 0, 8 * kMaxGroups, st));
    for (size_t g = 0; g < G; g++) {
      const int L = (int)s->groups[g].levels.size();
      if (k[g] >= L) continue;
      any = true;
      if (fsize[g] == 0 || s->groups[g].levels[k[g]].r == 0) {  // as run_levels: all deeper levels empty
        for (int kk = k[g]; kk < L; kk++) {
          LevelData& d = s->data[g][kk];
          d.rec = nullptr;
          d.n = 0;
          d.evals = (kk == k[g]) ? fsize[g] * (uint64_t)s->groups[g].levels[kk].r : 0;
          d.pairs = d.evals;
          if (kk > 0 && kk == k[g] && fsize[g] > 0) {
            atf_status e = ATF_OK;
            char* csr = arena_take(s, (int)g, (fsize[g] + 1) * 8, &e);
            if (!csr) return e ? e : fail(s, ATF_ERR_OOM, "csr");
            CUDA_TRY(s, cudaMemsetAsync(csr, 0, (fsize[g] + 1) * 8, st));
            s->data[g][kk - 1].csr = (uint64_t*)csr;
          }
        }
        k[g] = L;
        continue;
      }
      Pending pd;
      atf_status e;
      auto& T = s->tails[g];
      if (T.phase == 1) {
        if ((e = queue_tail_emit(s, (int)g, pd, active > 1))) return e;
        tails_done.push_back((int)g);
        k[g] = L;
      } else if (tail_here(s, (int)g, k[g], fsize[g])) {
        if ((e = queue_tail_count(s, (int)g, k[g], frontier[g], fsize[g], pd, active > 1))) return e;
        for (int d = 0; d < T.nl; d++) T.tot[d] = s->replay_f[g][k[g] + d];
        T.phase = 1;  // the emit is queued next round, sized from the expected totals
      } else {
        const uint64_t want = s->replay_f[g][k[g]];
        if ((e = queue_level(s, (int)g, k[g], frontier[g], fsize[g], pd, active > 1, want))) return e;
        GroupPlan& gp = s->groups[g];
        LevelData& d = s->data[g][k[g]];
        d.rec = pd.child;
        d.n = want;
        d.evals = fsize[g] * (uint64_t)gp.levels[k[g]].r;
        if (!(s->opts.flags & ATF_FLAG_TIMING)) d.pairs = 0;
        if (k[g] > 0) s->data[g][k[g] - 1].csr = pd.csr;
        expect.push_back(ReplayExpect{round, (int)g, want});
        if (s->opts.flags & ATF_FLAG_TIMING) timed.emplace_back((int)g, k[g]);
        frontier[g] = pd.child;
        fsize[g] = want;
        k[g]++;
      }
      pend.push_back(pd);
    }
    if (!any) break;
    for (auto& pd : pend)
      if (pd.joined) CUDA_TRY(s, cudaStreamWaitEvent(st, s->gb[pd.g].join, 0));
    if (!pend.empty())
      CUDA_TRY(s, cudaMemcpyAsync((char*)s->d_replay + (size_t)round * 12 * kMaxGroups, s->d_totals, 12 * kMaxGroups,
                                  cudaMemcpyDeviceToDevice, st));
  }
  rounds_out = round;
  return ATF_OK;
}

// One synchronisation, then every level total and overflow flag against the expected ones.
static atf_status replay_check(atf_space* s, int round, const std::vector<ReplayExpect>& expect,
                               const std::vector<std::pair<int, int>>& timed, const std::vector<int>& tails_done) {
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  // one synchronisation: the round log, then the checks
  std::vector<unsigned long long> log((size_t)round * 12 * kMaxGroups / 8 + 1, 0);
  if (round) CUDA_TRY(s, cudaMemcpyAsync(log.data(), s->d_replay, (size_t)round * 12 * kMaxGroups, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(s, cudaStreamSynchronize(st));
  for (const ReplayExpect& x : expect) {
    const unsigned long long* rl = log.data() + (size_t)x.round * 12 * kMaxGroups / 8;
    const unsigned int* ovf = reinterpret_cast<const unsigned int*>(rl + kMaxGroups);
    if (rl[x.g] != x.total || ovf[x.g]) return fail(s, ATF_ERR_STATE, "replay: level total differs (group %d)", x.g);
  }
  for (int g : tails_done) finish_tail(s, g);  // totals were the expected ones (tail scans)
  for (auto& gk : timed) {
    LevelData& d = s->data[gk.first][gk.second];
    cudaEventElapsedTime(&d.ms, s->events[gk.first][gk.second].first, s->events[gk.first][gk.second].second);
    cudaEventElapsedTime(&d.expand_ms, s->events[gk.first][gk.second].first, s->events[gk.first][gk.second].mid);
    d.pairs = d.evals;  // the headline flags; the segment-bound pair counts are not logged per level here
  }
  return ATF_OK;
}


static void replay_reset(atf_space* s) {
  const size_t G = s->groups.size();
  for (size_t g = 0; g < G; g++) {
    s->data[g].assign(s->groups[g].levels.size(), LevelData{});
    for (auto& c : s->arena[g]) c.used = 0;
  }
  s->tails.assign(G, {});
}

static atf_status run_levels_replay(atf_space* s) {
  NvtxRange nvtx("atf replay");
  cudaStream_t user_st = (cudaStream_t)s->opts.stream;
  const size_t G = s->groups.size();
  int max_rounds = 0;
  for (size_t g = 0; g < G; g++) max_rounds = std::max(max_rounds, (int)s->groups[g].levels.size() + 1);
  if ((size_t)max_rounds > s->replay_cap) {
    dfree(s, (char*)s->d_replay, s->replay_cap * 12 * kMaxGroups);
    s->replay_cap = (size_t)max_rounds;
    s->d_replay = (unsigned long long*)dalloc(s, s->replay_cap * 12 * kMaxGroups);
    if (!s->d_replay) { s->replay_cap = 0; return fail(s, ATF_ERR_OOM, "replay log"); }
  }
  auto& S = s->gsnap;
  if (s->graph_exec && s->graph_epoch == s->buf_epoch) {
    // the captured generation: its host-side state, then one graph launch
    NvtxRange nvtx_g("atf replay (graph)");
    s->data = S.data;
    for (size_t g = 0; g < G; g++)
      for (size_t i = 0; i < s->arena[g].size() && i < S.used[g].size(); i++) s->arena[g][i].used = S.used[g][i];
    s->tails = S.tails;
    CUDA_TRY(s, cudaGraphLaunch(s->graph_exec, user_st));
    s->replays++;
    return replay_check(s, S.rounds, S.expect, {}, S.tails_done);
  }
  if (s->graph_exec) {  // stale: a buffer it references moved
    cudaGraphExecDestroy(s->graph_exec);
    s->graph_exec = nullptr;
  }
  // the second replay in a row (every buffer sized by the first) is captured as a graph
  const bool capture = s->replays >= 1 && !(s->opts.flags & ATF_FLAG_TIMING);
  int rounds = 0;
  std::vector<ReplayExpect> expect;
  std::vector<std::pair<int, int>> timed;
  std::vector<int> tails_done;
  atf_status e = ATF_OK;
  bool captured = false;
  if (capture) {
    if (!s->cap_stream) CUDA_TRY(s, cudaStreamCreateWithFlags(&s->cap_stream, cudaStreamNonBlocking));
    if (!s->cap_ev) CUDA_TRY(s, cudaEventCreateWithFlags(&s->cap_ev, cudaEventDisableTiming));
    cudaGraph_t graph = nullptr;
    if (cudaStreamBeginCapture(s->cap_stream, cudaStreamCaptureModeThreadLocal) == cudaSuccess) {
      s->opts.stream = s->cap_stream;
      s->capturing = true;
      e = replay_queue(s, rounds, expect, timed, tails_done);
      const cudaError_t ce = cudaStreamEndCapture(s->cap_stream, &graph);
      s->capturing = false;
      s->opts.stream = user_st;
      if (e == ATF_OK && ce == cudaSuccess && graph &&
          cudaGraphInstantiate(&s->graph_exec, graph, 0) == cudaSuccess) {
        captured = true;
      } else {
        s->graph_exec = nullptr;
      }
      if (graph) cudaGraphDestroy(graph);
    }
    cudaGetLastError();
    if (captured) {
      S.data = s->data;
      S.used.assign(G, {});
      for (size_t g = 0; g < G; g++)
        for (auto& c : s->arena[g]) S.used[g].push_back(c.used);
      S.tails = s->tails;
      S.rounds = rounds;
      S.expect = expect;
      S.tails_done = tails_done;
      s->graph_epoch = s->buf_epoch;
      CUDA_TRY(s, cudaGraphLaunch(s->graph_exec, user_st));
    } else {  // not capturable (e.g. a buffer had to grow): the plain replay
      s->err.clear();
      replay_reset(s);
      rounds = 0;
      expect.clear();
      timed.clear();
      tails_done.clear();
    }
  }
  if (!captured) {
    e = replay_queue(s, rounds, expect, timed, tails_done);
    if (e) return e;
  }
  s->replays++;
  return replay_check(s, rounds, expect, timed, tails_done);
}

// ---------------------------------------------------------------- balanced multi-GPU generation
// SURVEY.md §8(e), DESIGN.md §6.  Every level is distributed afresh: rank r expands the parents
// [r F / N, (r + 1) F / N) of the previous level (F = its global size), so every rank evaluates
// the same number of (node, candidate) pairs at every level (f_{k-1} r_k / N), whatever the
// shape of the tree.  Rank r's children are a contiguous slice of the level in canonical order
// (children of a contiguous parent slice).  After each level round the ranks all-gather a small
// record per group (level counts + where the new level's records live), fix their CSR entries to
// global child indices, and copy their next parent slice from the owning ranks: CUDA IPC
// pointers (one process per GPU: peer memory over NVLink / NVSwitch) or plain pointers (ranks
// in one process).
static atf_status dist_desc(atf_space* s, int g, const uint32_t* rec, DistDesc& d) {
  std::memset(&d, 0, sizeof d);
  d.pid = (int64_t)getpid();
  if (!rec) return ATF_OK;
  for (auto& c : s->arena[g])
    if ((const char*)rec >= c.p && (const char*)rec < c.p + c.size) {
      d.base = (uint64_t)(uintptr_t)c.p;
      d.off = (uint64_t)((const char*)rec - c.p);
      if (!c.has_ipc) {  // exported once per allocation
        cudaIpcMemHandle_t h;
        CUDA_TRY(s, cudaIpcGetMemHandle(&h, c.p));
        std::memcpy(c.ipc, &h, sizeof h);
        c.has_ipc = true;
      }
      std::memcpy(d.handle, c.ipc, 64);
      return ATF_OK;
    }
  return fail(s, ATF_ERR_STATE, "internal: level records outside the arena");
}

static atf_status dist_peer_ptr(atf_space* s, int q, const DistDesc& d, const char** out) {
  if (d.pid == (int64_t)getpid()) {  // ranks in one process (tests, the one-GPU prediction)
    *out = (const char*)(uintptr_t)d.base + d.off;
    return ATF_OK;
  }
  for (auto& pm : s->peers)
    if (pm.rank == q && std::memcmp(pm.handle, d.handle, 64) == 0) {
      *out = pm.base + d.off;
      return ATF_OK;
    }
  cudaIpcMemHandle_t h;
  std::memcpy(&h, d.handle, sizeof h);
  void* p = nullptr;
  CUDA_TRY(s, cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
  atf_space::PeerMap pm;
  pm.rank = q;
  std::memcpy(pm.handle, d.handle, 64);
  pm.base = (char*)p;
  s->peers.push_back(pm);
  *out = pm.base + d.off;
  return ATF_OK;
}

// This rank's round-flag array (allocated and exported once per space).
static atf_status dist_flags_desc(atf_space* s, DistDesc& d) {
  std::memset(&d, 0, sizeof d);
  d.pid = (int64_t)getpid();
  if (!s->d_dflags) {
    s->d_dflags = (unsigned long long*)dalloc(s, 8 * (kDistMaxRounds + 2));
    if (!s->d_dflags) return fail(s, ATF_ERR_OOM, "round flags");
    CUDA_TRY(s, cudaMemset(s->d_dflags, 0, 8 * (kDistMaxRounds + 2)));
    s->dist_epoch = 0;
    s->dflags_has_ipc = false;
  }
  if (!s->dflags_has_ipc) {
    cudaIpcMemHandle_t h;
    CUDA_TRY(s, cudaIpcGetMemHandle(&h, s->d_dflags));
    std::memcpy(s->dflags_ipc, &h, sizeof h);
    s->dflags_has_ipc = true;
  }
  d.base = (uint64_t)(uintptr_t)s->d_dflags;
  std::memcpy(d.handle, s->dflags_ipc, 64);
  return ATF_OK;
}

// Timing gate (ATF_FLAG_TIMING): hold the stream, queue, release (see host_gate_kernel).
static atf_status gate_hold(atf_space* s, cudaStream_t st) {
  if (!s->h_gate) {
    CUDA_TRY(s, cudaHostAlloc((void**)&s->h_gate, 64, cudaHostAllocMapped));
    CUDA_TRY(s, cudaHostGetDevicePointer((void**)&s->d_gate, s->h_gate, 0));
    *(volatile unsigned int*)s->h_gate = 0;
    s->gate_v = 0;
  }
  int ce = launch_host_gate(s->d_gate, ++s->gate_v, st);
  if (ce) return fail(s, ATF_ERR_CUDA, "timing gate");
  return ATF_OK;
}
static void gate_release(atf_space* s) {
  if (s->h_gate) {
    std::atomic_thread_fence(std::memory_order_seq_cst);
    *(volatile unsigned int*)s->h_gate = s->gate_v;
  }
}

// Group-to-rank assignment of the balanced generation.  Ranks are laid on a line
// of world * kCapU capacity units; group g owns the units [cap_lo, cap_lo + cap_n) and rank q
// expands the share of every level of g that its units [q kCapU, (q+1) kCapU) overlap.  With
// the previous generation's candidate pairs per group (identical on every rank), cap_n is
// proportional to them: every rank gets 1/world of the total work, and a rank works on one or
// two groups with slices of 1/(world * share) instead of every group at 1/world (fewer, larger
// kernels per round).  Without that information (first generation, one group, one rank)
// every group spans all ranks: cap_lo = 0, cap_n = world * kCapU (slices [rF/N, (r+1)F/N)).
constexpr uint64_t kCapU = 1ull << 20;
static void dist_assignment(const atf_space* s, int world, std::vector<uint64_t>& c, std::vector<uint64_t>& u) {
  const size_t G = s->groups.size();
  const uint64_t units = (uint64_t)world * kCapU;
  c.assign(G, 0);
  u.assign(G, units);
  double W = 0;
  for (double w : s->group_work) W += w;
  if ((s->opts.flags & ATF_FLAG_DIST_NO_SUBSETS) || world == 1 || G < 2 || s->group_work.size() != G || !(W > 0)) return;
  uint64_t used = 0;
  size_t big = 0;
  for (size_t g = 0; g < G; g++) {
    u[g] = std::max<uint64_t>(1, (uint64_t)(s->group_work[g] / W * (double)units));
    used += u[g];
    if (s->group_work[g] > s->group_work[big]) big = g;
  }
  if (used > units) {  // (only through the 1-unit minimum) shave the largest group
    u[big] -= std::min(u[big] - 1, used - units);
  } else {
    u[big] += units - used;
  }
  uint64_t at = 0;
  for (size_t g = 0; g < G; g++) {
    c[g] = at;
    at += u[g];
  }
}

// One balanced generation.  mode 0: synchronous rounds (sizes found on the device, one
// all-gather per round), recorded in s->dlog.  mode 1: the same with every level sized from the
// log (the allocation sequence -- hence every address a peer reads -- is the one mode 2 will
// reproduce); if every count matches, mode 2 is allowed next.  mode 2: no host synchronisation
// and no all-gather per round: counts, offsets and peer addresses come from the log, a rank
// publishes each round in its flag array and waits on the owners' flags before its peer copies;
// at the end every rank checks its level totals, overflow flags, wait time-outs and its own
// addresses against the log, and one all-gather of the verdicts decides for all ranks
// (ATF_ERR_STATE: regenerate with mode 0).
static atf_status generate_dist_pass(atf_space* s, int rank, int world, atf_allgather_fn ag, void* ctx, int mode,
                                     bool* verdict_done) {
  *verdict_done = false;
  NvtxRange nvtx(mode == 2 ? "atf_space_generate_dist (replay)" : "atf_space_generate_dist");
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  const size_t G = s->groups.size();
  auto& X = s->dlog;
  std::vector<int> k(G, 0);
  std::vector<uint64_t> F(G, 1);                 // global size of the frontier (level k - 1)
  std::vector<uint64_t> lo(G, 0), hi(G, 0);      // this rank's parent slice of the frontier
  std::vector<const uint32_t*> frontier(G, s->d_root);
  std::vector<DistGroup> mine(G), all((size_t)world * G);
  const size_t pay = sizeof(DistGroup) * G + sizeof(DistDesc);
  std::vector<char> sendb(pay), recvb(pay * world);
  DistDesc my_flags;
  atf_status e0 = dist_flags_desc(s, my_flags);
  if (e0) return e0;
  const bool timing = (s->opts.flags & ATF_FLAG_TIMING) != 0;
  std::vector<std::vector<DistGroup>> rec_all;   // this generation's per-round records (modes 0, 1)
  std::vector<char> rec_ex;
  std::vector<DistDesc> rec_fd;
  bool counts_match = mode == 1;
  bool bad = false;                              // mode 2: own address differs from the log
  struct Expect { int round, g; uint64_t total; };
  std::vector<Expect> expect;
  const unsigned long long epoch = mode == 2 ? ++s->dist_epoch : 0;
  if (timing && s->dist_ev.size() < 4 * (size_t)kDistMaxRounds) {
    for (auto ev : s->dist_ev) cudaEventDestroy(ev);
    s->dist_ev.assign(4 * kDistMaxRounds, nullptr);
    for (auto& ev : s->dist_ev) CUDA_TRY(s, cudaEventCreate(&ev));
  }
  s->dist_round_ms.clear();
  if (mode == 2 && (size_t)kDistMaxRounds > s->replay_cap) {
    dfree(s, (char*)s->d_replay, s->replay_cap * 12 * kMaxGroups);
    s->replay_cap = kDistMaxRounds;
    s->d_replay = (unsigned long long*)dalloc(s, s->replay_cap * 12 * kMaxGroups);
    if (!s->d_replay) { s->replay_cap = 0; return fail(s, ATF_ERR_OOM, "replay log"); }
  }
  // Small levels are replicated: every rank expands the whole frontier while it costs less than
  // kReplEvals candidate pairs (no exchange, no copy; the first distributed level takes its
  // parent slice straight from the local copy).  C5: levels 1-3 replicated, 4-8 distributed.
  const uint64_t kReplEvals = 1ull << g_repl_log2.load();
  std::vector<char> repl(G, 1);
  std::vector<uint64_t> cap_lo, cap_n;
  dist_assignment(s, world, cap_lo, cap_n);
  if (mode >= 1 && (cap_lo != X.cap_lo || cap_n != X.cap_n)) return fail(s, ATF_ERR_STATE, "internal: assignment changed");
  bool subsets = false;  // some group does not span every rank
  for (size_t g = 0; g < G; g++) subsets |= cap_lo[g] != 0 || cap_n[g] != (uint64_t)world * kCapU;
  // this rank's share [l, h) of a level of group g with Fg nodes (empty: not a member of g)
  auto share = [&](size_t g, uint64_t Fg, uint64_t& l, uint64_t& h) {
    const uint64_t c = cap_lo[g], u = cap_n[g], q0 = (uint64_t)rank * kCapU, q1 = q0 + kCapU;
    const uint64_t a = std::max(c, q0), b = std::min(c + u, q1);
    if (b <= a) {
      l = h = 0;
      return false;
    }
    l = (uint64_t)((unsigned __int128)Fg * (a - c) / u);
    h = (uint64_t)((unsigned __int128)Fg * (b - c) / u);
    return true;
  };
  std::vector<char> member(G, 0);
  std::vector<double> work(G, 0.0);
  for (size_t g = 0; g < G; g++) {  // level 0: the root (one parent), expanded by the group's ranks
    uint64_t l, h;
    member[g] = share(g, 1, l, h) ? 1 : 0;
    lo[g] = 0;
    hi[g] = member[g] ? 1 : 0;
  }
  int round = 0;
  for (;; round++) {
    if (round >= kDistMaxRounds) return fail(s, ATF_ERR_STATE, "generate_dist: too many rounds");
    if (mode == 2 && round >= (int)X.all.size()) break;  // every logged round replayed (checked below)
    const DistGroup* logged = mode >= 1 && round < (int)X.all.size() ? X.all[round].data() + (size_t)rank * G : nullptr;
    char rname[48];
    snprintf(rname, sizeof rname, "atf dist round %d", round);
    NvtxRange nvtx_round(rname);
    if (timing) {
      atf_status e = gate_hold(s, st);
      if (e) return e;
      CUDA_TRY(s, cudaEventRecord(s->dist_ev[4 * round], st));
    }
    std::vector<Pending> pend;
    int active = 0;
    for (size_t g = 0; g < G; g++)
      if (k[g] < (int)s->groups[g].levels.size() && hi[g] > lo[g] && s->groups[g].levels[k[g]].r > 0) active++;
    bool any_open = false;
    for (size_t g = 0; g < G; g++) mine[g] = DistGroup{};
    for (int attempt = 0;; attempt++) {
      pend.clear();
      CUDA_TRY(s, cudaMemsetAsync(s->d_totals, 0, 16 * kMaxGroups, st));
      if (timing) CUDA_TRY(s, cudaMemsetAsync(s->d_pairs, 0, 8 * kMaxGroups, st));
      for (size_t g = 0; g < G; g++) {
        const int L = (int)s->groups[g].levels.size();
        if (k[g] >= L || mine[g].nd) continue;
        any_open = true;
        const uint64_t np = hi[g] - lo[g];
        const bool empty_range = s->groups[g].levels[k[g]].r == 0;
        if (np == 0 || empty_range) {
          // no local parents (or an empty range): this rank's part of the level is empty (and,
          // at the start of the group's fused tail, of every tail level: the ranks that have
          // parents complete the tail's levels in this round); the parents' CSR entries are 0
          const int nd = (!empty_range && s->tails[g].phase == 0 && tail_here(s, (int)g, k[g], F[g])) ? L - k[g] : 1;
          for (int d = 0; d < nd; d++) {
            LevelData& ld = s->data[g][k[g] + d];
            ld.rec = nullptr;
            ld.n = 0;
            ld.csr = nullptr;
            ld.evals = d == 0 ? np * (uint64_t)s->groups[g].levels[k[g]].r : 0;
            ld.pairs = ld.evals;
          }
          if (k[g] > 0) {
            atf_status e = ATF_OK;
            char* csr = arena_take(s, (int)g, (np + 1) * 8, &e);
            if (!csr) return e ? e : fail(s, ATF_ERR_OOM, "csr");
            CUDA_TRY(s, cudaMemsetAsync(csr, 0, (np + 1) * 8, st));
            LevelData& pdl = s->data[g][k[g] - 1];
            pdl.csr = (uint64_t*)csr;
            pdl.csr_offset = lo[g];
            pdl.csr_n = np;
          }
          mine[g].nd = (uint32_t)nd;
          for (int d = 0; d < nd; d++) mine[g].cnt[d] = 0;
          continue;
        }
        Pending pd;
        atf_status e;
        auto& T = s->tails[g];
        if (T.phase == 1) {
          e = queue_tail_emit(s, (int)g, pd, active > 1);
        } else if (tail_here(s, (int)g, k[g], F[g])) {
          e = queue_tail_count(s, (int)g, k[g], frontier[g], np, pd, active > 1);
          if (!e && mode == 2) {  // sizes from the log: the emit follows in the same queue
            if (!logged || logged[g].nd != (uint32_t)T.nl) return fail(s, ATF_ERR_STATE, "replay: tail log");
            for (int d = 0; d < T.nl; d++) T.tot[d] = logged[g].cnt[d];
            T.phase = 1;
            pend.push_back(pd);
            e = queue_tail_emit(s, (int)g, pd, active > 1);
          }
        } else {
          uint64_t want = UINT64_MAX;
          if (logged) {
            if (logged[g].nd != 1) {
              if (mode == 2) return fail(s, ATF_ERR_STATE, "replay: level log");
              counts_match = false;
            } else {
              want = logged[g].cnt[0];
            }
          }
          e = queue_level(s, (int)g, k[g], frontier[g], np, pd, active > 1, mode >= 1 ? want : UINT64_MAX);
          if (!e && mode == 2) {
            GroupPlan& gp = s->groups[g];
            LevelData& d = s->data[g][k[g]];
            d.rec = pd.child;
            d.n = want;
            d.evals = np * (uint64_t)gp.levels[k[g]].r;
            d.pairs = d.evals;
            if (k[g] > 0) {
              LevelData& pdl = s->data[g][k[g] - 1];
              pdl.csr = pd.csr;
              pdl.csr_offset = lo[g];
              pdl.csr_n = np;
            }
            expect.push_back(Expect{round, (int)g, want});
            mine[g].nd = 1;
            mine[g].cnt[0] = want;
          }
        }
        if (e) return e;
        pend.push_back(pd);
      }
      if (pend.empty()) break;
      for (auto& pd : pend)
        if (pd.joined) CUDA_TRY(s, cudaStreamWaitEvent(st, s->gb[pd.g].join, 0));
      if (mode == 2) {  // no synchronisation: the round's totals go to the device log
        CUDA_TRY(s, cudaMemcpyAsync((char*)s->d_replay + (size_t)round * 12 * kMaxGroups, s->d_totals,
                                    12 * kMaxGroups, cudaMemcpyDeviceToDevice, st));
        for (auto& pd : pend)
          if (pd.kind == 2) {
            const int g = pd.g;
            finish_tail(s, g);
            auto& T = s->tails[g];
            s->data[g][T.k0 > 0 ? T.k0 - 1 : 0].csr_offset = lo[g];
            if (T.k0 > 0) s->data[g][T.k0 - 1].csr_n = hi[g] - lo[g];
            mine[g].nd = (uint32_t)T.nl;
            for (int d = 0; d < T.nl; d++) mine[g].cnt[d] = T.tot[d];
          }
        break;
      }
      CUDA_TRY(s, cudaMemcpyAsync(s->h_ctl.data(), s->d_totals, 12 * kMaxGroups, cudaMemcpyDeviceToHost, st));
      for (auto& pd : pend)
        if (pd.kind == 1) {
          auto& T = s->tails[pd.g];
          for (int d = 0; d < T.nl; d++)
            CUDA_TRY(s, cudaMemcpyAsync(&T.tot[d], T.t.tile_base + d * (T.t.n_tiles + 1) + T.t.n_tiles, 8,
                                        cudaMemcpyDeviceToHost, st));
        }
      if (timing) gate_release(s);
      CUDA_TRY(s, cudaStreamSynchronize(st));
      unsigned long long h_pairs[kMaxGroups] = {};
      if (timing) CUDA_TRY(s, cudaMemcpy(h_pairs, s->d_pairs, sizeof(h_pairs), cudaMemcpyDeviceToHost));
      bool redo = false;
      for (auto& pd : pend) {
        const int g = pd.g;
        if (pd.kind == 1) {  // tail counted: its emit runs in the same round (sizes known)
          s->tails[g].phase = 1;
          redo = true;
          continue;
        }
        if (pd.kind == 2) {
          finish_tail(s, g);
          auto& T = s->tails[g];
          s->data[g][T.k0 > 0 ? T.k0 - 1 : 0].csr_offset = lo[g];
          if (T.k0 > 0) s->data[g][T.k0 - 1].csr_n = hi[g] - lo[g];
          mine[g].nd = (uint32_t)T.nl;
          for (int d = 0; d < T.nl; d++) mine[g].cnt[d] = T.tot[d];
          continue;
        }
        const uint64_t total = s->h_totals[g];
        GroupPlan& gp = s->groups[g];
        if (s->h_flags[g] || total > pd.cap) {  // overflow: grow and redo within this round
          counts_match = false;
          s->stash_hint = std::max<uint64_t>(s->stash_hint, total);
          atf_status e = arena_grow(s, g, total * gp.words * 4 + (pd.n_parents + 1) * 8);
          if (e) return e;
          redo = true;
          continue;
        }
        Chunk& c = s->arena[g][pd.chunk];
        c.used = pd.child_off + ((total * gp.words * 4 + 255) & ~(uint64_t)255);
        LevelData& d = s->data[g][pd.k];
        d.rec = pd.child;
        d.n = total;
        d.evals = pd.n_parents * (uint64_t)gp.levels[pd.k].r;
        if (pd.k > 0) {
          LevelData& pdl = s->data[g][pd.k - 1];
          pdl.csr = pd.csr;
          pdl.csr_offset = lo[g];
          pdl.csr_n = pd.n_parents;
        }
        if (timing) {
          cudaEventElapsedTime(&d.ms, s->events[g][pd.k].first, s->events[g][pd.k].second);
          cudaEventElapsedTime(&d.expand_ms, s->events[g][pd.k].first, s->events[g][pd.k].mid);
          d.pairs = d.seg_skip ? h_pairs[g] : d.evals;
        }
        mine[g].nd = 1;
        mine[g].cnt[0] = total;
      }
      if (!redo) break;
    }
    if (!any_open) break;
    if (timing) CUDA_TRY(s, cudaEventRecord(s->dist_ev[4 * round + 1], st));  // (synchronised above)
    // exchange: one record per group and rank (skipped when every completed level is replicated:
    // all ranks take that decision from the same global sizes)
    bool need_ag = false;
    for (size_t g = 0; g < G; g++) {
      mine[g].repl = repl[g];
      // (with subsets, the non-members of a group learn its replicated levels' sizes here too)
      if (mine[g].nd && (!repl[g] || subsets)) need_ag = true;
      if (mine[g].nd != 1 || repl[g]) continue;
      atf_status e = dist_desc(s, (int)g, s->data[g][k[g]].rec, mine[g].desc);
      if (e) return e;
    }
    if (mode == 2) {
      if ((bool)X.exchanged[round] != need_ag) return fail(s, ATF_ERR_STATE, "replay: round structure");
      all = X.all[round];
      for (size_t g = 0; g < G; g++) {  // peers read what the log says this rank wrote
        const DistGroup& lg = all[(size_t)rank * G + g];
        if (lg.nd != mine[g].nd || (mine[g].nd == 1 && !repl[g] &&
                                    (lg.desc.base != mine[g].desc.base || lg.desc.off != mine[g].desc.off)))
          bad = true;
      }
    } else if (need_ag) {
      std::memcpy(sendb.data(), mine.data(), sizeof(DistGroup) * G);
      std::memcpy(sendb.data() + sizeof(DistGroup) * G, &my_flags, sizeof(DistDesc));
      if (ag(sendb.data(), recvb.data(), pay, ctx) != 0)
        return fail(s, ATF_ERR_CUDA, "all-gather callback failed in round %d", round);
      for (int r = 0; r < world; r++) {
        std::memcpy(all.data() + (size_t)r * G, recvb.data() + pay * r, sizeof(DistGroup) * G);
        if (rec_fd.empty() || (int)rec_fd.size() < world) {
          DistDesc fd;
          std::memcpy(&fd, recvb.data() + pay * r + sizeof(DistGroup) * G, sizeof fd);
          if ((int)rec_fd.size() == r) rec_fd.push_back(fd);
        }
      }
    } else {
      for (int r = 0; r < world; r++)
        for (size_t g = 0; g < G; g++) all[(size_t)r * G + g] = mine[g];
    }
    if (mode != 2) {
      if (mode == 1) {  // same counts as the log on every rank?
        if (round >= (int)X.all.size() || (bool)X.exchanged[round] != need_ag) {
          counts_match = false;
        } else {
          for (size_t i = 0; i < all.size() && counts_match; i++) {
            const DistGroup &x = all[i], &y = X.all[round][i];
            if (x.nd != y.nd || std::memcmp(x.cnt, y.cnt, sizeof x.cnt) != 0) counts_match = false;
          }
        }
      }
      rec_all.push_back(all);
      rec_ex.push_back(need_ag ? 1 : 0);
    }
    // bookkeeping and CSR fix-ups of every group, then (replay) this rank's round flag, then the
    // peer copies: a rank publishes its round before it waits on anyone's
    if (timing) {
      atf_status e = gate_hold(s, st);
      if (e) return e;
      CUDA_TRY(s, cudaEventRecord(s->dist_ev[4 * round + 2], st));
    }
    struct Copy { int g; };
    std::vector<int> copy_groups;
    for (size_t g = 0; g < G; g++) {
      const uint32_t nd = mine[g].nd;
      if (!nd) continue;
      for (int r = 0; r < world; r++)
        if (all[(size_t)r * G + g].nd != nd) return fail(s, ATF_ERR_STATE, "ranks out of step (group %zu)", g);
      if (repl[g]) {  // every rank of the group holds the whole level(s)
        for (uint32_t d = 0; d < nd; d++) {
          LevelData& ld = s->data[g][k[g] + d];
          ld.offset = 0;
          if (d + 1 < nd) { ld.csr_offset = 0; ld.csr_n = ld.n; }
          uint64_t fg = 0;  // the members' count (non-members hold none)
          for (int r = 0; r < world; r++) fg = std::max<uint64_t>(fg, all[(size_t)r * G + g].cnt[d]);
          work[g] += (double)F[g] * (double)s->groups[g].levels[k[g] + d].r;
          F[g] = fg;
        }
        k[g] += (int)nd;
        if (k[g] >= (int)s->groups[g].levels.size()) continue;
        const uint64_t Fg = F[g];
        const LevelData& ld = s->data[g][k[g] - 1];
        if (Fg * (uint64_t)s->groups[g].levels[k[g]].r >= kReplEvals) {
          repl[g] = 0;  // distribute from here on: this rank's slice of the local copy
          share(g, Fg, lo[g], hi[g]);
        } else {
          lo[g] = 0;
          hi[g] = member[g] ? Fg : 0;
        }
        frontier[g] = (ld.rec && hi[g] > lo[g]) ? ld.rec + lo[g] * s->groups[g].words : s->d_root;
        continue;
      }
      // global offsets of this rank's part of every completed level; CSR entries -> global
      for (uint32_t d = 0; d < nd; d++) {
        uint64_t before = 0, tot = 0;
        for (int r = 0; r < world; r++) {
          const uint64_t c = all[(size_t)r * G + g].cnt[d];
          if (r < rank) before += c;
          tot += c;
        }
        LevelData& ld = s->data[g][k[g] + d];
        ld.offset = before;
        if (d + 1 < nd) {  // a tail's inner level: its CSR (this rank's nodes) came with it
          ld.csr_offset = before;
          ld.csr_n = ld.n;
        }
        // the CSR of the level above points into this rank's local child array
        LevelData* pl = k[g] + (int)d > 0 ? &s->data[g][k[g] + d - 1] : nullptr;
        if (pl && pl->csr && before) {
          int ce = launch_add_offset(pl->csr, pl->csr_n + 1, before, st);
          if (ce) return fail(s, ATF_ERR_CUDA, "csr fix-up");
        }
        work[g] += (double)F[g] * (double)s->groups[g].levels[k[g] + d].r;
        F[g] = tot;
      }
      k[g] += (int)nd;
      const int L = (int)s->groups[g].levels.size();
      if (k[g] >= L) continue;
      share(g, F[g], lo[g], hi[g]);
      if (hi[g] > lo[g]) copy_groups.push_back((int)g);
    }
    if (mode == 2 && need_ag && world > 1) {
      int ce = launch_dist_flag_set(s->d_dflags + round, epoch, st);
      if (ce) return fail(s, ATF_ERR_CUDA, "round flag");
    }
    std::vector<char> waited(world, 0);
    for (int g : copy_groups) {
      // the next parent slice, copied from the ranks holding it
      const uint64_t np = hi[g] - lo[g];
      const int W = s->groups[g].words;
      auto& gbf = s->gb[g];
      atf_status e = ensure_buf(s, &gbf.pbuf, &gbf.pbuf_cap, np * W * 4, "parent slice");
      if (e) return e;
      uint64_t pos = 0;  // global index of records[0] of rank q
      for (int q = 0; q < world; q++) {
        const DistGroup& dg = all[(size_t)q * G + g];
        const uint64_t n = dg.cnt[0], a0 = std::max(pos, lo[g]), a1 = std::min(pos + n, hi[g]);
        if (a1 > a0) {
          const char* src = nullptr;
          if ((e = dist_peer_ptr(s, q, dg.desc, &src))) return e;
          if (mode == 2 && q != rank && !waited[q]) {  // the owner's round is complete
            const char* fp = nullptr;
            if ((e = dist_peer_ptr(s, q, X.flag_desc[q], &fp))) return e;
            int ce = launch_dist_flag_wait((const unsigned long long*)fp + round, epoch,
                                           s->d_dflags + kDistMaxRounds, st);
            if (ce) return fail(s, ATF_ERR_CUDA, "round flag wait");
            waited[q] = 1;
          }
          CUDA_TRY(s, cudaMemcpyAsync(gbf.pbuf + (a0 - lo[g]) * W * 4, src + (a0 - pos) * W * 4, (a1 - a0) * W * 4,
                                      cudaMemcpyDeviceToDevice, st));
        }
        pos += n;
      }
      frontier[g] = (const uint32_t*)gbf.pbuf;
    }
    if (timing) {
      CUDA_TRY(s, cudaEventRecord(s->dist_ev[4 * round + 3], st));
      gate_release(s);
    }
  }
  s->gsize.assign(G, 0);
  for (size_t g = 0; g < G; g++) s->gsize[g] = s->groups[g].levels.empty() ? 0 : (k[g] >= (int)s->groups[g].levels.size() ? F[g] : 0);
  s->shard_rank = rank;
  s->shard_world = world;
  s->group_work = work;
  if (mode == 2) {
    // one synchronisation, then the checks, then one all-gather of the verdicts
    std::vector<unsigned long long> log((size_t)round * 12 * kMaxGroups / 8 + 1, 0);
    unsigned long long werr = 0;
    if (round) CUDA_TRY(s, cudaMemcpyAsync(log.data(), s->d_replay, (size_t)round * 12 * kMaxGroups, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(s, cudaMemcpyAsync(&werr, s->d_dflags + kDistMaxRounds, 8, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(s, cudaStreamSynchronize(st));
    bool ok = !bad && werr == 0 && round == (int)X.all.size();
    for (const Expect& x : expect) {
      const unsigned long long* rl = log.data() + (size_t)x.round * 12 * kMaxGroups / 8;
      const unsigned int* ovf = reinterpret_cast<const unsigned int*>(rl + kMaxGroups);
      if (rl[x.g] != x.total || ovf[x.g]) ok = false;
    }
    if (werr) CUDA_TRY(s, cudaMemset(s->d_dflags + kDistMaxRounds, 0, 8));
    int32_t mine_ok = ok ? 1 : 0;
    std::vector<int32_t> oks(world, 0);
    *verdict_done = true;
    if (ag(&mine_ok, oks.data(), sizeof(int32_t), ctx) != 0) return fail(s, ATF_ERR_CUDA, "all-gather callback failed (replay check)");
    for (int r = 0; r < world; r++)
      if (!oks[r]) return fail(s, ATF_ERR_STATE, "generate_dist replay: rank %d's checks failed", r);
  } else {
    if ((int)rec_fd.size() < world) {  // no exchange took place (world 1 or all levels replicated)
      rec_fd.assign(world, my_flags);
    }
    X.world = world;
    X.rank = rank;
    X.G = G;
    X.flags = s->opts.flags;
    X.all = std::move(rec_all);
    X.exchanged = std::move(rec_ex);
    X.flag_desc = std::move(rec_fd);
    X.cap_lo = cap_lo;
    X.cap_n = cap_n;
    X.pure_ok = mode == 1 && counts_match;
  }
  if (timing) {
    CUDA_TRY(s, cudaStreamSynchronize(st));
    for (int r = 0; r < round; r++) {  // the round's kernels + its fix-ups and peer copies (not the
      float a = 0.f, b = 0.f;         // host wait for the all-gather in between)
      cudaEventElapsedTime(&a, s->dist_ev[4 * r], s->dist_ev[4 * r + 1]);
      cudaEventElapsedTime(&b, s->dist_ev[4 * r + 2], s->dist_ev[4 * r + 3]);
      s->dist_round_ms.push_back(a + b);
    }
  }
  s->state = FINAL_SHARD;
  return ATF_OK;
}

static void dist_reset(atf_space* s) {
  const size_t G = s->groups.size();
  s->data.assign(G, {});
  s->tails.assign(G, {});
  for (size_t g = 0; g < G; g++) {
    s->data[g].assign(s->groups[g].levels.size(), LevelData{});
    for (auto& c : s->arena[g]) c.used = 0;
  }
}

// Mode choice (generate_dist_pass): replay once a synchronous generation with the same ranks,
// flags and log-sized levels reproduced every count; a failed replay (all ranks learn it from
// the verdict all-gather) is regenerated synchronously at once.
static atf_status generate_dist_impl(atf_space* s, int rank, int world, atf_allgather_fn ag, void* ctx) {
  auto& X = s->dlog;
  std::vector<uint64_t> cl, cn;
  dist_assignment(s, world, cl, cn);
  const bool same = X.world == world && X.rank == rank && X.G == s->groups.size() && X.flags == s->opts.flags &&
                    !X.all.empty() && cl == X.cap_lo && cn == X.cap_n;
  const bool replay_allowed = !(s->opts.flags & (ATF_FLAG_NO_REPLAY | ATF_FLAG_TIMING));
  const int mode = (same && replay_allowed) ? (X.pure_ok ? 2 : 1) : 0;
  bool verdict = false;
  atf_status e = generate_dist_pass(s, rank, world, ag, ctx, mode, &verdict);
  if (mode != 2 || e == ATF_OK) return e;
  if (!verdict) {  // failed before the checks: drain, then tell the other ranks
    cudaStreamSynchronize((cudaStream_t)s->opts.stream);
    cudaGetLastError();
    int32_t zero = 0;
    std::vector<int32_t> oks(world, 0);
    if (ag(&zero, oks.data(), sizeof(int32_t), ctx) != 0) return fail(s, ATF_ERR_CUDA, "all-gather callback failed (replay check)");
  }
  X.pure_ok = false;
  X.all.clear();
  dist_reset(s);
  return generate_dist_pass(s, rank, world, ag, ctx, 0, &verdict);
}

static atf_status generate_impl(atf_space* s) {
  NvtxRange nvtx("atf_space_generate");
  s->dlog.all.clear();  // a balanced generation's log describes arena contents this one replaces
  s->dlog.pure_ok = false;
  s->decode_jit = nullptr;  // the decoder's immediates (group sizes) belong to one generation
  s->decode_jit_tried = false;
  atf_status e = plan(s);
  if (e) return e;
  if ((e = ensure_device(s))) return e;
  size_t G = s->groups.size();
  s->data.assign(G, {});
  s->tails.assign(G, {});
  for (size_t g = 0; g < G; g++) {
    s->data[g].assign(s->groups[g].levels.size(), LevelData{});
    for (auto& c : s->arena[g]) c.used = 0;
  }
  if (s->opts.flags & ATF_FLAG_TIMING) {
    if (s->events.size() != G) {
      s->events.assign(G, {});
      for (size_t g = 0; g < G; g++) {
        s->events[g].resize(s->groups[g].levels.size());
        for (auto& ev : s->events[g]) {
          CUDA_TRY(s, cudaEventCreate(&ev.first));
          CUDA_TRY(s, cudaEventCreate(&ev.mid));
          CUDA_TRY(s, cudaEventCreate(&ev.second));
        }
      }
    }
  }
  bool replayed = false;
  // (not with ATF_FLAG_TIMING: the timing pass keeps one synchronisation per round so that the
  // per-level statistics, segment-bound pair counts included, are read as the levels complete)
  if (s->replay_ok && !(s->opts.flags & (ATF_FLAG_NO_REPLAY | ATF_FLAG_TIMING))) {
    e = run_levels_replay(s);
    if (e == ATF_OK) {
      replayed = true;
    } else {  // sizes differ from the recorded ones: regenerate level by level
      cudaStreamSynchronize((cudaStream_t)s->opts.stream);
      cudaGetLastError();
      s->replay_ok = false;
      drop_graph(s);
      for (size_t g = 0; g < G; g++) {
        s->data[g].assign(s->groups[g].levels.size(), LevelData{});
        for (auto& c : s->arena[g]) c.used = 0;
      }
      s->tails.assign(G, {});
    }
  }
  if (!replayed) {
    std::vector<int> gs(G), kf(G, 0);
    std::iota(gs.begin(), gs.end(), 0);
    std::vector<const uint32_t*> fr(G, s->d_root);
    std::vector<uint64_t> fz(G, 1);
    if (G > 1 && g_async_rounds.load() && !(s->opts.flags & (ATF_FLAG_TIMING | ATF_FLAG_SERIAL_GROUPS))) {
      if ((e = run_levels_async(s))) return e;
    } else if ((e = run_levels(s, gs, kf, fr, fz))) {
      return e;
    }
    s->replay_f.assign(G, {});
    for (size_t g = 0; g < G; g++)
      for (auto& d : s->data[g]) s->replay_f[g].push_back(d.n);
    s->replay_ok = true;
  }
  s->gsize.assign(G, 0);
  for (size_t g = 0; g < G; g++) s->gsize[g] = s->groups[g].levels.empty() ? 0 : s->data[g].back().n;
  s->group_work.assign(G, 0.0);  // candidate pairs per group (generate_dist's assignment)
  for (size_t g = 0; g < G; g++) {
    uint64_t f = 1;
    for (size_t k = 0; k < s->data[g].size(); k++) {
      s->group_work[g] += (double)f * (double)s->groups[g].levels[k].r;
      f = s->data[g][k].n;
    }
  }
  s->state = GENERATED;
  return ATF_OK;
}

// ---------------------------------------------------------------- checkpoint / resume
// A generated space on disk (SURVEY.md §5 "Checkpoint / resume: serialise spec + level arrays"):
// the spec (names, int64 range values in range order, constraint programs) and every group's
// level arrays (path records, CSR), so a tuning run resumes without regenerating.  Loading
// re-plans the spec (deterministic: same groups and record layout, checked against the file)
// and uploads the arrays.  Little-endian; FNV-1a 64 checksum of everything before it.
static const char kCkptMagic[8] = {'A', 'T', 'F', 'S', 'P', 'C', '0', '1'};
constexpr uint32_t kCkptVersion = 1;

namespace {
struct CkWriter {
  FILE* f;
  uint64_t h = 1469598103934665603ull;
  bool ok = true;
  void put(const void* p, size_t n) {
    const unsigned char* b = (const unsigned char*)p;
    for (size_t i = 0; i < n; i++) h = (h ^ b[i]) * 1099511628211ull;
    if (n && std::fwrite(p, 1, n, f) != n) ok = false;
  }
  template <typename T> void val(T v) { put(&v, sizeof v); }
};
struct CkReader {
  FILE* f;
  uint64_t h = 1469598103934665603ull;
  bool ok = true;
  bool get(void* p, size_t n) {
    if (!ok || (n && std::fread(p, 1, n, f) != n)) return ok = false;
    const unsigned char* b = (const unsigned char*)p;
    for (size_t i = 0; i < n; i++) h = (h ^ b[i]) * 1099511628211ull;
    return true;
  }
  template <typename T> bool val(T& v) { return get(&v, sizeof v); }
};
}  // namespace

atf_status atf_space_save(const atf_space* cs, const char* path) {
  atf_space* s = (atf_space*)cs;
  if (!s || !path) return ATF_ERR_INVALID_ARG;
  if (s->state != GENERATED) return fail(s, ATF_ERR_STATE, "save needs a generated (non-shard) space");
  for (size_t g = 0; g < s->groups.size(); g++)
    for (auto& d : s->data[g])
      if (d.offset != 0 || (d.csr_n != UINT64_MAX && d.csr_n != d.n))
        return fail(s, ATF_ERR_STATE, "save: the space holds a rank's part of a distributed generation");
  CUDA_TRY(s, cudaSetDevice(s->opts.device));
  CUDA_TRY(s, cudaStreamSynchronize((cudaStream_t)s->opts.stream));
  FILE* f = std::fopen(path, "wb");
  if (!f) return fail(s, ATF_ERR_INVALID_ARG, "cannot open %s for writing", path);
  CkWriter w{f};
  w.put(kCkptMagic, 8);
  w.val<uint32_t>(kCkptVersion);
  w.val<uint32_t>((uint32_t)s->params.size());
  for (auto& p : s->params) {
    w.val<uint32_t>((uint32_t)p.name.size());
    w.put(p.name.data(), p.name.size());
    const uint64_t n = p.values.size();
    w.val<uint64_t>(n);
    for (uint64_t j = 0; j < n; j++) w.val<int64_t>(p.v64 ? p.values64[j] : (int64_t)p.values[j]);
    w.val<uint32_t>((uint32_t)p.programs.size());
    for (auto& prog : p.programs) {
      w.val<uint32_t>((uint32_t)prog.size());
      w.put(prog.data(), prog.size() * 4);
    }
  }
  w.val<uint32_t>((uint32_t)s->groups.size());
  std::vector<char> buf;
  atf_status st = ATF_OK;
  for (size_t g = 0; g < s->groups.size() && st == ATF_OK && w.ok; g++) {
    const GroupPlan& gp = s->groups[g];
    w.val<uint32_t>((uint32_t)gp.levels.size());
    w.val<uint32_t>((uint32_t)gp.words);
    for (size_t k = 0; k < gp.levels.size() && w.ok; k++) {
      const LevelData& d = s->data[g][k];
      const uint64_t n = d.rec ? d.n : 0;
      const uint64_t nc = (k + 1 < gp.levels.size() && d.csr && n) ? n + 1 : 0;
      w.val<uint64_t>(n);
      w.val<uint64_t>(nc);
      const size_t rb = (size_t)n * gp.words * 4, cb = (size_t)nc * 8;
      buf.resize(std::max<size_t>(rb, cb) + 1);
      if (rb) {
        if (cudaMemcpy(buf.data(), d.rec, rb, cudaMemcpyDeviceToHost) != cudaSuccess) { st = ATF_ERR_CUDA; break; }
        w.put(buf.data(), rb);
      }
      if (cb) {
        if (cudaMemcpy(buf.data(), d.csr, cb, cudaMemcpyDeviceToHost) != cudaSuccess) { st = ATF_ERR_CUDA; break; }
        w.put(buf.data(), cb);
      }
    }
  }
  const uint64_t h = w.h;
  if (st == ATF_OK) w.put(&h, 8);
  const bool ok = w.ok && std::fclose(f) == 0;
  if (st != ATF_OK) return fail(s, st, "save: device copy failed: %s", cudaGetErrorString(cudaGetLastError()));
  if (!ok) return fail(s, ATF_ERR_INVALID_ARG, "save: write to %s failed", path);
  return ATF_OK;
}

static atf_status load_impl(atf_space* s, FILE* f) {
  CkReader r{f};
  char magic[8];
  uint32_t ver = 0, np = 0;
  if (!r.get(magic, 8) || std::memcmp(magic, kCkptMagic, 8) != 0) return fail(s, ATF_ERR_INVALID_ARG, "load: not an atfgen checkpoint");
  if (!r.val(ver) || ver != kCkptVersion) return fail(s, ATF_ERR_INVALID_ARG, "load: unsupported checkpoint version");
  if (!r.val(np) || np > ATF_MAX_PARAMS) return fail(s, ATF_ERR_INVALID_ARG, "load: bad parameter count");
  for (uint32_t p = 0; p < np; p++) {
    uint32_t nl = 0;
    if (!r.val(nl) || nl == 0 || nl > 4096) return fail(s, ATF_ERR_INVALID_ARG, "load: bad name");
    std::string name(nl, '\0');
    uint64_t n = 0;
    if (!r.get(&name[0], nl) || !r.val(n) || n > ATF_MAX_RANGE) return fail(s, ATF_ERR_INVALID_ARG, "load: bad range");
    std::vector<int64_t> vals(n);
    if (n && !r.get(vals.data(), n * 8)) return fail(s, ATF_ERR_INVALID_ARG, "load: truncated range");
    atf_range rg{};
    rg.kind = ATF_RANGE_SET64;
    rg.values64 = vals.data();
    rg.n_values = (int64_t)n;
    int32_t id = -1;
    atf_status e = atf_space_add_param(s, name.c_str(), &rg, &id);
    if (e) return e;
    uint32_t nprog = 0;
    if (!r.val(nprog) || nprog > 1024) return fail(s, ATF_ERR_INVALID_ARG, "load: bad program count");
    for (uint32_t q = 0; q < nprog; q++) {
      uint32_t nw = 0;
      if (!r.val(nw) || nw == 0 || nw > ATF_MAX_PROGRAM_WORDS) return fail(s, ATF_ERR_INVALID_ARG, "load: bad program");
      std::vector<int32_t> code(nw);
      if (!r.get(code.data(), nw * 4)) return fail(s, ATF_ERR_INVALID_ARG, "load: truncated program");
      if ((e = atf_space_add_constraint(s, id, code.data(), (int32_t)nw))) return e;
    }
  }
  atf_status e = plan(s);
  if (e) return e;
  uint32_t G = 0;
  if (!r.val(G) || G != s->groups.size()) return fail(s, ATF_ERR_INVALID_ARG, "load: group structure differs from the plan");
  if ((e = ensure_device(s))) return e;
  s->data.assign(G, {});
  s->tails.assign(G, {});
  std::vector<char> buf;
  for (uint32_t g = 0; g < G; g++) {
    const GroupPlan& gp = s->groups[g];
    uint32_t L = 0, W = 0;
    if (!r.val(L) || !r.val(W) || L != gp.levels.size() || W != (uint32_t)gp.words)
      return fail(s, ATF_ERR_INVALID_ARG, "load: level layout of group %u differs from the plan", g);
    s->data[g].assign(L, LevelData{});
    uint64_t above = 1;
    for (uint32_t k = 0; k < L; k++) {
      uint64_t n = 0, nc = 0;
      if (!r.val(n) || !r.val(nc)) return fail(s, ATF_ERR_INVALID_ARG, "load: truncated level");
      if (n > above * (uint64_t)gp.levels[k].r || (nc && nc != n + 1) || (nc && k + 1 == L))
        return fail(s, ATF_ERR_INVALID_ARG, "load: inconsistent level sizes");
      LevelData& d = s->data[g][k];
      d.n = n;
      d.evals = above * (uint64_t)gp.levels[k].r;
      const size_t rb = (size_t)n * W * 4, cb = (size_t)nc * 8;
      buf.resize(std::max<size_t>(rb, cb) + 1);
      if (rb) {
        if (!r.get(buf.data(), rb)) return fail(s, ATF_ERR_INVALID_ARG, "load: truncated records");
        char* p = arena_take(s, (int)g, rb, &e);
        if (!p) return e ? e : fail(s, ATF_ERR_OOM, "load: records");
        CUDA_TRY(s, cudaMemcpy(p, buf.data(), rb, cudaMemcpyHostToDevice));
        d.rec = (uint32_t*)p;
      }
      if (cb) {
        if (!r.get(buf.data(), cb)) return fail(s, ATF_ERR_INVALID_ARG, "load: truncated CSR");
        char* p = arena_take(s, (int)g, cb, &e);
        if (!p) return e ? e : fail(s, ATF_ERR_OOM, "load: CSR");
        CUDA_TRY(s, cudaMemcpy(p, buf.data(), cb, cudaMemcpyHostToDevice));
        d.csr = (uint64_t*)p;
      }
      above = n;
    }
  }
  const uint64_t want = r.h;
  uint64_t got = 0;
  if (!r.get(&got, 8) || got != want) return fail(s, ATF_ERR_INVALID_ARG, "load: checksum mismatch");
  s->gsize.assign(G, 0);
  s->group_work.assign(G, 0.0);
  for (uint32_t g = 0; g < G; g++) {
    s->gsize[g] = s->groups[g].levels.empty() ? 0 : s->data[g].back().n;
    uint64_t fr = 1;
    for (size_t k = 0; k < s->data[g].size(); k++) {
      s->group_work[g] += (double)fr * (double)s->groups[g].levels[k].r;
      fr = s->data[g][k].n;
    }
  }
  s->replay_ok = false;  // a later generate recomputes level by level
  s->state = GENERATED;
  return ATF_OK;
}

atf_status atf_space_load(const atf_space_opts* opts, const char* path, atf_space** out) {
  if (!out || !path) return ATF_ERR_INVALID_ARG;
  *out = nullptr;
  atf_space* s = nullptr;
  atf_status e = atf_space_create(opts, &s);
  if (e) return e;
  FILE* f = std::fopen(path, "rb");
  if (!f) {
    e = fail(s, ATF_ERR_INVALID_ARG, "cannot open %s", path);
  } else {
    e = load_impl(s, f);
    std::fclose(f);
  }
  *out = s;  // also on error: atf_space_last_error(s) says why; the caller destroys it
  return e;
}

// ---------------------------------------------------------------- decode args
static atf_status make_decode_args(const atf_space* s, DecodeArgs& a) {
  std::memset(&a, 0, sizeof a);
  a.n_groups = (int)s->groups.size();
  a.n_params = (int)s->params.size();
  int l = 0;
  for (int g = 0; g < a.n_groups; g++) {
    const GroupPlan& gp = s->groups[g];
    a.gsize[g] = s->gsize[g];
    a.gmagic[g] = s->gsize[g] ? ~0ull / s->gsize[g] : 0ull;
    a.leaves[g] = s->data[g].back().rec;
    a.words[g] = gp.words;
    a.lvl_begin[g] = l;
    for (auto& lp : gp.levels) {
      a.lvl_param[l] = (int16_t)lp.param;
      a.lvl_word[l] = (int16_t)lp.field_word;
      a.lvl_shift[l] = (int16_t)lp.field_shift;
      a.lvl_bits[l] = (int16_t)lp.field_bits;
      a.lvl_range[l] = s->d_range[lp.param];
      a.lvl_range64[l] = s->d_range64[lp.param];
      l++;
    }
  }
  a.lvl_begin[a.n_groups] = l;
  return ATF_OK;
}

// ---------------------------------------------------------------- shard host logic
// S§8(e).  Rank `rank` of `world` takes the contiguous slice [lo, hi) of the cut level
// whose child-count prefix (csr[0..ncut], csr[ncut] = T children) lies in
// [rank*T/world, (rank+1)*T/world): contiguity keeps each rank's leaves a contiguous range
// of the canonical order; balancing by children evens out the expansion below the cut.
static void shard_slice(const uint64_t* csr, uint64_t ncut, int rank, int world, uint64_t* lo, uint64_t* hi) {
  const uint64_t T = csr[ncut];
  auto bound = [&](int r_) -> uint64_t {  // first cut node whose child prefix >= r T / world
    u128 target = (u128)T * (u128)r_ / (u128)world;
    return (uint64_t)(std::lower_bound(csr, csr + ncut + 1, (uint64_t)target) - csr);
  };
  *lo = rank == 0 ? 0 : std::min<uint64_t>(bound(rank), ncut);
  *hi = rank == world - 1 ? ncut : std::min<uint64_t>(bound(rank + 1), ncut);
  if (*hi < *lo) *hi = *lo;
}
// all: [world][n] per-rank counts (rank-major).  Entry idx: the global offset of rank's
// part (exclusive scan over ranks) and the global total.
static void shard_offsets(const int64_t* all, int world, int n, int idx, int rank, uint64_t* before,
                          uint64_t* tot) {
  *before = 0;
  *tot = 0;
  for (int r = 0; r < world; r++) {
    const uint64_t c = (uint64_t)all[(size_t)r * n + idx];
    if (r < rank) *before += c;
    *tot += c;
  }
}

// ================================================================= C ABI
extern "C" {

const char* atf_status_str(atf_status st) {
  switch (st) {
    case ATF_OK: return "ok";
    case ATF_ERR_INVALID_ARG: return "invalid argument";
    case ATF_ERR_OOM: return "out of memory";
    case ATF_ERR_CUDA: return "CUDA error";
    case ATF_ERR_STATE: return "invalid state";
    case ATF_ERR_BYTECODE: return "bad bytecode";
    case ATF_ERR_FORWARD_REF: return "forward reference";
    case ATF_ERR_OVERFLOW: return "overflow";
    case ATF_ERR_INDEX: return "index out of range";
    case ATF_ERR_DUPLICATE: return "duplicate";
    case ATF_ERR_LIMIT: return "limit exceeded";
  }
  return "unknown";
}

const char* atf_space_last_error(const atf_space* s) { return s ? s->err.c_str() : "null space"; }

atf_status atf_space_create(const atf_space_opts* opts, atf_space** out) {
  if (!out) return ATF_ERR_INVALID_ARG;
  atf_space* s = new (std::nothrow) atf_space();
  if (!s) return ATF_ERR_OOM;
  if (opts) s->opts = *opts;
  if (s->opts.alloc && !s->opts.free) {
    delete s;
    return ATF_ERR_INVALID_ARG;
  }
  *out = s;
  return ATF_OK;
}

atf_status atf_space_add_param(atf_space* s, const char* name, const atf_range* range, int32_t* out_id) {
  if (!s || !name || !range) return fail(s, ATF_ERR_INVALID_ARG, "null argument");
  if (s->state != BUILDING) return fail(s, ATF_ERR_STATE, "add_param after plan/generate");
  if (!*name) return fail(s, ATF_ERR_INVALID_ARG, "empty name");
  if (s->params.size() >= ATF_MAX_PARAMS) return fail(s, ATF_ERR_LIMIT, "more than %d parameters", ATF_MAX_PARAMS);
  for (auto& p : s->params)
    if (p.name == name) return fail(s, ATF_ERR_DUPLICATE, "duplicate parameter name %s (P:53: unique)", name);
  ParamDef pd;
  pd.name = name;
  // P:57 ranges; readings #1-#3, #5, #22 (values materialised in int64)
  std::vector<int64_t> vals;
  if (range->kind == ATF_RANGE_INTERVAL || range->kind == ATF_RANGE_POW2) {
    if (range->step <= 0) return fail(s, ATF_ERR_INVALID_ARG, "step must be positive");
    if (range->end >= range->begin) {
      i128 count = ((i128)range->end - range->begin) / range->step + 1;
      if (count > ATF_MAX_RANGE) return fail(s, ATF_ERR_LIMIT, "range of %s has more than 2^24 values", name);
    }
    for (i128 i = range->begin; i <= range->end; i += range->step) {
      if (range->kind == ATF_RANGE_INTERVAL) {
        vals.push_back((int64_t)i);
      } else {
        if (i < 0 || i > 62) return fail(s, ATF_ERR_INVALID_ARG, "pow2 exponent outside [0,62]");
        vals.push_back((int64_t)1 << (int)i);
      }
    }
  } else if (range->kind == ATF_RANGE_GEN) {
    // P:57 generator over i: the program is checked like a constraint (no PARAM) and
    // evaluated exactly in int64 for every i
    if (range->step <= 0) return fail(s, ATF_ERR_INVALID_ARG, "step must be positive");
    if (range->n_values <= 0 || range->n_values > ATF_MAX_PROGRAM_WORDS || !range->values)
      return fail(s, ATF_ERR_BYTECODE, "generator of %s: bad program length", name);
    const int32_t* code = range->values;
    const int n = (int)range->n_values;
    for (int i = 0; i < n;) {
      const int op = code[i];
      if (op == ATF_OP_PARAM) return fail(s, ATF_ERR_BYTECODE, "generator of %s references a parameter", name);
      if (op < ATF_OP_X || op > ATF_OP_NOT) return fail(s, ATF_ERR_BYTECODE, "generator of %s: bad opcode", name);
      i += op == ATF_OP_CONST ? 3 : 1;
      if (i > n) return fail(s, ATF_ERR_BYTECODE, "generator of %s: truncated CONST", name);
    }
    if (range->end >= range->begin) {
      i128 count = ((i128)range->end - range->begin) / range->step + 1;
      if (count > ATF_MAX_RANGE) return fail(s, ATF_ERR_LIMIT, "range of %s has more than 2^24 values", name);
    }
    for (i128 i = range->begin; i <= range->end; i += range->step) {
      if (i < INT64_MIN || i > INT64_MAX) return fail(s, ATF_ERR_INVALID_ARG, "generator index outside int64");
      int64_t st[ATF_MAX_STACK + 1];
      int sp = 0;
      bool poison = false, bad = false;
      for (int k = 0; k < n && !bad;) {
        const int op = code[k];
        if (op == ATF_OP_X || op == ATF_OP_CONST) {
          if (sp >= ATF_MAX_STACK) { bad = true; break; }
          st[sp++] = op == ATF_OP_X ? (int64_t)i
                                    : (int64_t)(((uint64_t)(uint32_t)code[k + 2] << 32) | (uint32_t)code[k + 1]);
          k += op == ATF_OP_X ? 1 : 3;
          continue;
        }
        if (op == ATF_OP_NOT) {
          if (sp < 1) { bad = true; break; }
          st[sp - 1] = st[sp - 1] == 0;
          k++;
          continue;
        }
        if (sp < 2) { bad = true; break; }
        const int64_t b = st[--sp], a = st[sp - 1];
        i128 r = 0;
        switch (op) {
          case ATF_OP_ADD: r = (i128)a + b; break;
          case ATF_OP_SUB: r = (i128)a - b; break;
          case ATF_OP_MUL: r = (i128)a * b; break;
          case ATF_OP_DIV: if (b == 0) poison = true; else r = (i128)a / b; break;     // C truncation
          case ATF_OP_MOD: if (b == 0) poison = true; else r = (i128)a % b; break;
          case ATF_OP_MIN: r = a < b ? a : b; break;
          case ATF_OP_MAX: r = a > b ? a : b; break;
          case ATF_OP_EQ: r = a == b; break;
          case ATF_OP_NE: r = a != b; break;
          case ATF_OP_LT: r = a < b; break;
          case ATF_OP_LE: r = a <= b; break;
          case ATF_OP_GT: r = a > b; break;
          case ATF_OP_GE: r = a >= b; break;
          case ATF_OP_DIVIDES: if (a == 0) poison = true; else r = ((i128)b % a) == 0; break;
          case ATF_OP_MULOF: if (b == 0) poison = true; else r = ((i128)a % b) == 0; break;
          case ATF_OP_AND: r = (a != 0) && (b != 0); break;
          case ATF_OP_OR: r = (a != 0) || (b != 0); break;
          default: bad = true;
        }
        if (r < INT64_MIN || r > INT64_MAX) return fail(s, ATF_ERR_OVERFLOW, "generator of %s overflows int64", name);
        st[sp - 1] = (int64_t)r;
        k++;
      }
      if (bad || sp != 1) return fail(s, ATF_ERR_BYTECODE, "generator of %s: malformed program", name);
      if (poison) return fail(s, ATF_ERR_BYTECODE, "generator of %s: zero divisor at i = %lld", name, (long long)i);
      vals.push_back(st[0]);
    }
    std::vector<int64_t> sorted(vals);
    std::sort(sorted.begin(), sorted.end());
    if (std::adjacent_find(sorted.begin(), sorted.end()) != sorted.end())
      return fail(s, ATF_ERR_DUPLICATE, "generator of %s repeats a value", name);
  } else if (range->kind == ATF_RANGE_SET || range->kind == ATF_RANGE_SET64) {
    const bool w = range->kind == ATF_RANGE_SET64;
    if (range->n_values < 0 || (range->n_values > 0 && !(w ? (const void*)range->values64 : (const void*)range->values)))
      return fail(s, ATF_ERR_INVALID_ARG, "bad set");
    if (range->n_values > ATF_MAX_RANGE) return fail(s, ATF_ERR_LIMIT, "set larger than 2^24");
    for (int64_t j = 0; j < range->n_values; j++) vals.push_back(w ? range->values64[j] : (int64_t)range->values[j]);
    std::vector<int64_t> sorted(vals);
    std::sort(sorted.begin(), sorted.end());
    if (std::adjacent_find(sorted.begin(), sorted.end()) != sorted.end())
      return fail(s, ATF_ERR_DUPLICATE, "duplicate value in set of %s", name);
  } else {
    return fail(s, ATF_ERR_INVALID_ARG, "unknown range kind %d", range->kind);
  }
  // int32 parameter: the values; int64 parameter: positions + the int64 table (reading #22)
  for (int64_t v : vals)
    if (v < INT32_MIN || v > INT32_MAX) pd.v64 = true;
  if (pd.v64) {
    pd.values64 = vals;
    pd.values.resize(vals.size());
    std::iota(pd.values.begin(), pd.values.end(), 0);
  } else {
    pd.values.assign(vals.begin(), vals.end());
  }
  if (!vals.empty()) {
    pd.vmin = *std::min_element(vals.begin(), vals.end());
    pd.vmax = *std::max_element(vals.begin(), vals.end());
  }
  s->params.push_back(std::move(pd));
  if (out_id) *out_id = (int32_t)s->params.size() - 1;
  return ATF_OK;
}

atf_status atf_space_add_constraint(atf_space* s, int32_t pid, const int32_t* code, int32_t n) {
  if (!s || !code) return fail(s, ATF_ERR_INVALID_ARG, "null argument");
  if (s->state != BUILDING) return fail(s, ATF_ERR_STATE, "add_constraint after plan/generate");
  if (pid < 0 || pid >= (int)s->params.size()) return fail(s, ATF_ERR_INVALID_ARG, "no parameter %d", pid);
  atf_status st = validate_program(s, pid, code, n);
  if (st) return st;
  s->params[pid].programs.emplace_back(code, code + n);
  return ATF_OK;
}

atf_status atf_space_plan(atf_space* s) {
  if (!s) return ATF_ERR_INVALID_ARG;
  if (s->state == BUILDING) {
    // static int64 interval analysis of every program (reading #9)
    for (size_t p = 0; p < s->params.size(); p++)
      for (auto& code : s->params[p].programs) {
        Tree t;
        std::string why;
        Iv xiv{s->params[p].vmin, s->params[p].vmax};
        if (parse_program(code, s->params, xiv, t, &why) < 0)
          return fail(s, ATF_ERR_OVERFLOW, "parameter %s: %s", s->params[p].name.c_str(), why.c_str());
      }
  }
  return plan(s);
}

atf_status atf_space_num_params(const atf_space* s, int32_t* out) {
  if (!s || !out) return ATF_ERR_INVALID_ARG;
  *out = (int32_t)s->params.size();
  return ATF_OK;
}

atf_status atf_space_param_name(const atf_space* s, int32_t p, char* buf, size_t cap, size_t* len_out) {
  if (!s || p < 0 || p >= (int32_t)s->params.size() || (!buf && cap)) return ATF_ERR_INVALID_ARG;
  const std::string& n = s->params[p].name;
  if (len_out) *len_out = n.size();
  if (cap) {
    const size_t m = std::min(cap - 1, n.size());
    std::memcpy(buf, n.data(), m);
    buf[m] = '\0';
  }
  return ATF_OK;
}

atf_status atf_space_num_groups(const atf_space* s, int32_t* out) {
  if (!s || !out) return ATF_ERR_INVALID_ARG;
  if (s->state == BUILDING) return ATF_ERR_STATE;
  *out = (int32_t)s->groups.size();
  return ATF_OK;
}

atf_status atf_space_group_members(const atf_space* s, int32_t g, int32_t* out, int32_t cap, int32_t* n_out) {
  if (!s || !n_out) return ATF_ERR_INVALID_ARG;
  if (s->state == BUILDING) return ATF_ERR_STATE;
  if (g < 0 || g >= (int)s->groups.size()) return ATF_ERR_INVALID_ARG;
  auto& m = s->groups[g].members;
  *n_out = (int32_t)m.size();
  for (int i = 0; i < (int)m.size() && i < cap && out; i++) out[i] = m[i];
  return ATF_OK;
}

atf_status atf_space_plan_json(const atf_space* s, char* buf, size_t cap, size_t* len_out) {
  if (!s) return ATF_ERR_INVALID_ARG;
  if (s->state == BUILDING) return ATF_ERR_STATE;
  std::string j = "{\"groups\":[";
  for (size_t g = 0; g < s->groups.size(); g++) {
    auto& gp = s->groups[g];
    j += (g ? "," : "") + std::string("{\"members\":[");
    for (size_t i = 0; i < gp.members.size(); i++) j += (i ? "," : "") + std::to_string(gp.members[i]);
    j += "],\"words\":" + std::to_string(gp.words) + ",\"levels\":[";
    for (size_t l = 0; l < gp.levels.size(); l++) {
      auto& lp = gp.levels[l];
      std::string d;
      for (char c : lp.desc) {
        if (c == '"' || c == '\\') d += '\\';
        d += c;
      }
      char tmp[256];
      snprintf(tmp, sizeof tmp,
               "{\"param\":%d,\"r\":%d,\"word\":%d,\"shift\":%d,\"bits\":%d,\"cost\":%.1f,\"generic\":%s,"
               "\"n_terms\":%d,\"n_gates\":%d,\"n_slots\":%d,\"qmax\":%u,\"desc\":\"",
               lp.param, lp.r, lp.field_word, lp.field_shift, lp.field_bits, lp.cost, lp.generic ? "true" : "false",
               lp.proto.n_terms, lp.proto.n_gates, lp.proto.n_slots, lp.proto.qmax);
      j += (l ? "," : "") + std::string(tmp) + d + "\"";
      j += ",\"terms\":[";
      for (int t = 0; t < lp.proto.n_terms; t++) {
        const Term& T = lp.proto.terms[t];
        snprintf(tmp, sizeof tmp, "%s{\"kind\":%d,\"variant\":%d,\"rel\":%d,\"qtable\":%d}", t ? "," : "", T.kind,
                 T.variant, T.rel, T.use_qtable);
        j += tmp;
      }
      j += "]}";
    }
    j += "]}";
  }
  j += "]}";
  if (len_out) *len_out = j.size();
  if (buf && cap > 0) {
    size_t n = std::min(cap - 1, j.size());
    memcpy(buf, j.data(), n);
    buf[n] = 0;
  }
  return ATF_OK;
}

atf_status atf_space_generate(atf_space* s) {
  if (!s) return ATF_ERR_INVALID_ARG;
  if (s->state == SHARDED) return fail(s, ATF_ERR_STATE, "space holds an unfinalized shard");
  if (s->dev_ready && s->ipc_alloc) release_device(s);  // back to the configured allocator
  s->ipc_alloc = false;
  if (s->state == BUILDING) {
    atf_status e = atf_space_plan(s);
    if (e) return e;
  }
  return generate_impl(s);
}

atf_status atf_space_size(const atf_space* s, uint64_t* lo, uint64_t* hi) {
  if (!s || !lo || !hi) return ATF_ERR_INVALID_ARG;
  if (s->state != GENERATED && s->state != FINAL_SHARD) return ATF_ERR_STATE;
  u128 S = 1;
  for (uint64_t z : s->gsize) {
    if (z && S > (~(u128)0) / z) return fail((atf_space*)s, ATF_ERR_OVERFLOW, "S >= 2^128");
    S *= z;
  }
  *lo = (uint64_t)S;
  *hi = (uint64_t)(S >> 64);
  return ATF_OK;
}

atf_status atf_space_group_size(const atf_space* s, int32_t g, uint64_t* out) {
  if (!s || !out) return ATF_ERR_INVALID_ARG;
  if (s->state != GENERATED && s->state != FINAL_SHARD) return ATF_ERR_STATE;
  if (g < 0 || g >= (int)s->groups.size()) return ATF_ERR_INVALID_ARG;
  *out = s->gsize[g];
  return ATF_OK;
}

atf_status atf_space_num_levels(const atf_space* s, int32_t g, int32_t* out) {
  if (!s || !out) return ATF_ERR_INVALID_ARG;
  if (s->state == BUILDING) return ATF_ERR_STATE;
  if (g < 0 || g >= (int)s->groups.size()) return ATF_ERR_INVALID_ARG;
  *out = (int32_t)s->groups[g].levels.size();
  return ATF_OK;
}

atf_status atf_space_level_size(const atf_space* s, int32_t g, int32_t k, uint64_t* out) {
  if (!s || !out) return ATF_ERR_INVALID_ARG;
  if (s->state < GENERATED) return ATF_ERR_STATE;
  if (g < 0 || g >= (int)s->groups.size() || k < 0 || k >= (int)s->groups[g].levels.size())
    return ATF_ERR_INVALID_ARG;
  *out = s->data[g][k].n;
  return ATF_OK;
}

atf_status atf_space_level_view(const atf_space* s, int32_t g, int32_t k, atf_level_view* out) {
  if (!s || !out) return ATF_ERR_INVALID_ARG;
  if (s->state < GENERATED) return ATF_ERR_STATE;
  if (g < 0 || g >= (int)s->groups.size() || k < 0 || k >= (int)s->groups[g].levels.size())
    return ATF_ERR_INVALID_ARG;
  const LevelData& d = s->data[g][k];
  const LevelPlan& lp = s->groups[g].levels[k];
  out->records = d.rec;
  out->csr = (k + 1 < (int)s->groups[g].levels.size()) ? d.csr : nullptr;
  out->n_nodes = d.n;
  out->offset = d.offset;
  out->words = s->groups[g].words;
  out->param = lp.param;
  out->field_word = lp.field_word;
  out->field_shift = lp.field_shift;
  out->field_bits = lp.field_bits;
  // the CSR covers this rank's nodes of level k (single GPU / generate_shard) or the parent slice
  // it expanded (generate_dist)
  out->csr_offset = d.csr_n != UINT64_MAX ? d.csr_offset : d.offset;
  out->csr_nodes = d.csr_n != UINT64_MAX ? d.csr_n : d.n;
  return ATF_OK;
}

static bool space_v64(const atf_space* s) {
  for (auto& p : s->params)
    if (p.v64) return true;
  return false;
}

// out: int32 SoA, or int64 SoA when w64 (reading #22; the int32 decoders refuse int64 spaces)
static atf_status decode_common(const atf_space* cs, const uint64_t* idx, const uint64_t* digits, int64_t n,
                                void* out, int64_t ld, void* stream, bool w64 = false) {
  atf_space* s = (atf_space*)cs;
  if (!s || (!idx && !digits) || !out || n < 0 || ld < n) return fail(s, ATF_ERR_INVALID_ARG, "bad decode arguments");
  if (s->state != GENERATED) return fail(s, ATF_ERR_STATE, "decode needs a generated (non-shard) space");
  if (!w64 && space_v64(s)) return fail(s, ATF_ERR_OVERFLOW, "values outside int32: use the *_i64 decoders");
  if (idx) {
    u128 S = 1;
    for (uint64_t z : s->gsize) S *= z;
    if (S >> 64) return fail(s, ATF_ERR_OVERFLOW, "S >= 2^64: use atf_space_decode_digits");
  }
  if (n == 0) return ATF_OK;
  CUDA_TRY(s, cudaSetDevice(s->opts.device));
  cudaStream_t st = (cudaStream_t)(stream ? stream : s->opts.stream);
  DecodeArgs a;
  make_decode_args(s, a);
  CUDA_TRY(s, cudaMemsetAsync(s->d_bad, 0, 4, st));
  // large batches: the decoder specialised for this space (NVRTC, compiled once per space)
  if (!w64 && n >= (1 << 18) && !(s->opts.flags & ATF_FLAG_NO_JIT) && !s->decode_jit_tried) {
    s->decode_jit = jit_decode_kernel(a);
    s->decode_jit_tried = true;
  }
  // random leaf gathers: ask for 32-byte L2 fetches for this launch (the default granularity
  // fetches a whole line per 8-byte record)
  size_t gran = 0;
  const bool big = n >= (1 << 18);
  if (big && cudaDeviceGetLimit(&gran, cudaLimitMaxL2FetchGranularity) == cudaSuccess && gran != 32)
    cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, 32);
  cudaGetLastError();
  int ce = (!w64 && big && s->decode_jit && !(s->opts.flags & ATF_FLAG_NO_JIT))
               ? jit_decode_launch(s->decode_jit, a, idx, digits, n, (int32_t*)out, ld, s->d_bad, st)
               : (idx ? launch_decode_indices(a, idx, n, out, w64 ? 1 : 0, ld, s->d_bad, st)
                      : launch_decode_digits(a, digits, n, out, w64 ? 1 : 0, ld, s->d_bad, st));
  if (big && gran && gran != 32) cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, gran);
  cudaGetLastError();
  if (ce) return fail(s, ATF_ERR_CUDA, "decode launch: %s", cudaGetErrorString((cudaError_t)ce));
  // the bad-index flag is read back only when someone could be out of range: always
  // check (one 4-byte copy) — it costs a sync, so the flag copy is async and we
  // synchronise the stream here to report ATF_ERR_INDEX deterministically.
  CUDA_TRY(s, cudaMemcpyAsync(s->h_flags, s->d_bad, 4, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(s, cudaStreamSynchronize(st));
  if (s->h_flags[0])
    return fail(s, ATF_ERR_INDEX, "index/digit out of range (rows set to %s)", w64 ? "INT64_MIN" : "INT32_MIN");
  return ATF_OK;
}

static void make_encode_args(const atf_space* s, EncodeArgs& a) {
  std::memset(&a, 0, sizeof a);
  a.n_groups = (int)s->groups.size();
  int l = 0;
  for (int g = 0; g < a.n_groups; g++) {
    const GroupPlan& gp = s->groups[g];
    a.gsize[g] = s->gsize[g];
    a.lvl_begin[g] = l;
    for (size_t k = 0; k < gp.levels.size(); k++, l++) {
      const LevelPlan& lp = gp.levels[k];
      const LevelData& d = s->data[g][k];
      a.lvl_param[l] = (int16_t)lp.param;
      a.lvl_word[l] = (int16_t)lp.field_word;
      a.lvl_shift[l] = (int16_t)lp.field_shift;
      a.lvl_bits[l] = (int16_t)lp.field_bits;
      a.lvl_words[l] = gp.words;
      a.lvl_rec[l] = d.rec;
      a.lvl_csr[l] = d.csr;
      a.lvl_n[l] = d.rec ? d.n : 0;
      a.lvl_sorted[l] = s->d_sorted[lp.param];
      a.lvl_r[l] = (int32_t)s->params[lp.param].values.size();
    }
  }
  a.lvl_begin[a.n_groups] = l;
  a.n_params = (int)s->params.size();
  for (int g = 0; g < a.n_groups; g++)
    for (int m : s->groups[g].members) a.param_group[m] = g;
  for (int p = 0; p < a.n_params; p++) {
    a.param_r[p] = (int32_t)s->params[p].values.size();
    a.param_range[p] = s->d_range[p];
  }
}

static atf_status encode_common(const atf_space* cs, const int32_t* vals, int64_t n, int64_t ld, uint64_t* digits,
                                uint64_t* idx, void* stream) {
  atf_space* s = (atf_space*)cs;
  if (!s || !vals || !digits || n < 0 || ld < n) return fail(s, ATF_ERR_INVALID_ARG, "bad encode arguments");
  if (s->state != GENERATED) return fail(s, ATF_ERR_STATE, "encode needs a generated (non-shard) space");
  if (space_v64(s)) return fail(s, ATF_ERR_LIMIT, "encode takes int32 configurations (int64 space)");
  if (idx) {
    u128 S = 1;
    for (uint64_t z : s->gsize) S *= z;
    if (S >> 64) return fail(s, ATF_ERR_OVERFLOW, "S >= 2^64: use atf_space_encode_digits");
  }
  if (n == 0) return ATF_OK;
  EncodeArgs a;
  make_encode_args(s, a);
  CUDA_TRY(s, cudaSetDevice(s->opts.device));
  cudaStream_t st = (cudaStream_t)(stream ? stream : s->opts.stream);
  int ce = launch_encode(a, vals, ld, n, digits, idx, st);
  if (ce) return fail(s, ATF_ERR_CUDA, "encode launch: %s", cudaGetErrorString((cudaError_t)ce));
  return ATF_OK;
}

atf_status atf_space_filter_product(atf_space* s, uint64_t* h_count, uint64_t* h_tuples) {
  if (!s || !h_count) return ATF_ERR_INVALID_ARG;
  atf_status e = plan(s);  // validation + static analysis (the product path needs no tree)
  if (e) return e;
  if (space_v64(s)) return fail(s, ATF_ERR_LIMIT, "the full-product filter takes int32 values (int64 space)");
  {
    u128 prod = 1;
    for (auto& p : s->params) prod *= (u128)p.values.size();
    if (prod >> 64) return fail(s, ATF_ERR_OVERFLOW, "full product >= 2^64");
  }
  if ((e = ensure_device(s))) return e;
  ProductArgs a;
  std::memset(&a, 0, sizeof a);
  a.n_params = (int)s->params.size();
  u128 total = 1;
  std::vector<int32_t> code, progs;
  for (int p = 0; p < a.n_params; p++) {
    const ParamDef& pd = s->params[p];
    a.r[p] = (int32_t)pd.values.size();
    a.range[p] = s->d_range[p];
    total *= (u128)pd.values.size();
    // the parameter's programs (ANDed), PARAM j -> SLOT j (slots = the tuple's values)
    a.prog_first[p] = (int32_t)progs.size() / 2;
    a.prog_count[p] = (int32_t)pd.programs.size();
    for (const auto& pr : pd.programs) {
      progs.push_back((int32_t)code.size());
      for (size_t i = 0; i < pr.size();) {
        const int op = pr[i];
        if (op == ATF_OP_PARAM) { code.push_back(OP_SLOT); code.push_back(pr[i + 1]); i += 2; }
        else if (op == ATF_OP_CONST) { code.insert(code.end(), pr.begin() + i, pr.begin() + i + 3); i += 3; }
        else { code.push_back(op); i += 1; }
      }
      progs.push_back((int32_t)code.size() - progs.back());
    }
  }
  if (total >> 64) return fail(s, ATF_ERR_OVERFLOW, "full product >= 2^64");
  a.total = (uint64_t)total;
  if (h_tuples) *h_tuples = a.total;
  if (a.total == 0) { *h_count = 0; return ATF_OK; }
  a.chunk = std::max<uint64_t>(1, std::min<uint64_t>(4096, a.total / (148ull * 2048)));
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  const size_t cbytes = std::max<size_t>(16, (code.size() + progs.size()) * 4);
  int32_t* d_code = (int32_t*)dalloc(s, cbytes);
  unsigned long long* d_cnt = (unsigned long long*)dalloc(s, 16);
  if (!d_code || !d_cnt) {
    dfree(s, d_code, cbytes);
    dfree(s, d_cnt, 16);
    return fail(s, ATF_ERR_OOM, "product filter scratch");
  }
  a.code = d_code;
  a.progs = d_code + code.size();
  std::vector<int32_t> up(code);
  up.insert(up.end(), progs.begin(), progs.end());
  atf_status out = ATF_OK;
  if (!up.empty() && cudaMemcpyAsync(d_code, up.data(), up.size() * 4, cudaMemcpyHostToDevice, st) != cudaSuccess)
    out = fail(s, ATF_ERR_CUDA, "product filter upload");
  if (!out && cudaMemsetAsync(d_cnt, 0, 8, st) != cudaSuccess) out = fail(s, ATF_ERR_CUDA, "memset");
  if (!out) {
    int ce = launch_filter_product(a, d_cnt, st);
    if (ce) out = fail(s, ATF_ERR_CUDA, "product filter launch: %s", cudaGetErrorString((cudaError_t)ce));
  }
  if (!out && (cudaMemcpyAsync(s->h_totals, d_cnt, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
               cudaStreamSynchronize(st) != cudaSuccess))
    out = fail(s, ATF_ERR_CUDA, "product filter readback");
  if (!out) *h_count = s->h_totals[0];
  dfree(s, d_code, cbytes);
  dfree(s, d_cnt, 16);
  return out;
}

atf_status atf_space_neighbors(const atf_space* cs, const int32_t* d_in, int64_t ld_in, int64_t n, uint64_t seed,
                               int32_t max_tries, int32_t* d_out, int64_t ld_out, int32_t* d_moved, void* stream) {
  atf_space* s = (atf_space*)cs;
  if (!s || !d_in || !d_out || !d_moved || n < 0 || ld_in < n || ld_out < n || max_tries < 0)
    return fail(s, ATF_ERR_INVALID_ARG, "bad neighbour arguments");
  if (s->state != GENERATED) return fail(s, ATF_ERR_STATE, "neighbours need a generated (non-shard) space");
  if (space_v64(s)) return fail(s, ATF_ERR_LIMIT, "neighbours take int32 configurations (int64 space)");
  if (n == 0) return ATF_OK;
  EncodeArgs a;
  make_encode_args(s, a);
  CUDA_TRY(s, cudaSetDevice(s->opts.device));
  cudaStream_t st = (cudaStream_t)(stream ? stream : s->opts.stream);
  int ce = launch_neighbors(a, d_in, ld_in, d_out, ld_out, n, seed, max_tries, d_moved, st);
  if (ce) return fail(s, ATF_ERR_CUDA, "neighbour launch: %s", cudaGetErrorString((cudaError_t)ce));
  return ATF_OK;
}

atf_status atf_space_encode_indices(const atf_space* s, const int32_t* d_values, int64_t n, int64_t ld,
                                    uint64_t* d_digits, uint64_t* d_idx, void* stream) {
  if (!d_idx) return fail((atf_space*)s, ATF_ERR_INVALID_ARG, "null index output");
  return encode_common(s, d_values, n, ld, d_digits, d_idx, stream);
}

atf_status atf_space_encode_digits(const atf_space* s, const int32_t* d_values, int64_t n, int64_t ld,
                                   uint64_t* d_digits, void* stream) {
  return encode_common(s, d_values, n, ld, d_digits, nullptr, stream);
}

atf_status atf_space_decode_indices(const atf_space* s, const uint64_t* d_idx, int64_t n, int32_t* d_out, int64_t ld,
                                    void* stream) {
  if (!d_idx) return fail((atf_space*)s, ATF_ERR_INVALID_ARG, "null indices");
  return decode_common(s, d_idx, nullptr, n, d_out, ld, stream);
}

static atf_status decode128_common(const atf_space* cs, const uint64_t* lo, const uint64_t* hi, uint64_t first_lo,
                                   uint64_t first_hi, int64_t n, void* out, int64_t ld, void* stream, bool w64 = false) {
  atf_space* s = (atf_space*)cs;
  if (!s || !out || n < 0 || ld < n) return fail(s, ATF_ERR_INVALID_ARG, "bad decode arguments");
  if (s->state != GENERATED) return fail(s, ATF_ERR_STATE, "decode needs a generated (non-shard) space");
  if (!w64 && space_v64(s)) return fail(s, ATF_ERR_OVERFLOW, "values outside int32: use the *_i64 decoders");
  u128 S = 1;
  for (uint64_t z : s->gsize) {
    if (z && S > (~(u128)0) / z) return fail(s, ATF_ERR_OVERFLOW, "S >= 2^128");
    S *= z;
  }
  if (n == 0) return ATF_OK;
  CUDA_TRY(s, cudaSetDevice(s->opts.device));
  cudaStream_t st = (cudaStream_t)(stream ? stream : s->opts.stream);
  DecodeArgs a;
  make_decode_args(s, a);
  CUDA_TRY(s, cudaMemsetAsync(s->d_bad, 0, 4, st));
  int ce = launch_decode128(a, lo, hi, first_lo, first_hi, n, out, w64 ? 1 : 0, ld, s->d_bad, (uint64_t)S,
                            (uint64_t)(S >> 64), st);
  if (ce) return fail(s, ATF_ERR_CUDA, "decode launch: %s", cudaGetErrorString((cudaError_t)ce));
  CUDA_TRY(s, cudaMemcpyAsync(s->h_flags, s->d_bad, 4, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(s, cudaStreamSynchronize(st));
  if (s->h_flags[0])
    return fail(s, ATF_ERR_INDEX, "index out of range (rows set to %s)", w64 ? "INT64_MIN" : "INT32_MIN");
  return ATF_OK;
}

atf_status atf_space_decode_indices128(const atf_space* s, const uint64_t* d_idx_lo, const uint64_t* d_idx_hi,
                                       int64_t n, int32_t* d_out, int64_t ld, void* stream) {
  if (!d_idx_lo || !d_idx_hi) return fail((atf_space*)s, ATF_ERR_INVALID_ARG, "null indices");
  return decode128_common(s, d_idx_lo, d_idx_hi, 0, 0, n, d_out, ld, stream);
}

atf_status atf_space_decode_range(const atf_space* s, uint64_t first_lo, uint64_t first_hi, int64_t n, int32_t* d_out,
                                  int64_t ld, void* stream) {
  return decode128_common(s, nullptr, nullptr, first_lo, first_hi, n, d_out, ld, stream);
}

atf_status atf_space_decode_digits(const atf_space* s, const uint64_t* d_digits, int64_t n, int32_t* d_out,
                                   int64_t ld, void* stream) {
  if (!d_digits) return fail((atf_space*)s, ATF_ERR_INVALID_ARG, "null digits");
  return decode_common(s, nullptr, d_digits, n, d_out, ld, stream);
}

atf_status atf_space_decode_indices_i64(const atf_space* s, const uint64_t* d_idx, int64_t n, int64_t* d_out,
                                        int64_t ld, void* stream) {
  if (!d_idx) return fail((atf_space*)s, ATF_ERR_INVALID_ARG, "null indices");
  return decode_common(s, d_idx, nullptr, n, d_out, ld, stream, true);
}

atf_status atf_space_decode_digits_i64(const atf_space* s, const uint64_t* d_digits, int64_t n, int64_t* d_out,
                                       int64_t ld, void* stream) {
  if (!d_digits) return fail((atf_space*)s, ATF_ERR_INVALID_ARG, "null digits");
  return decode_common(s, nullptr, d_digits, n, d_out, ld, stream, true);
}

atf_status atf_space_decode_range_i64(const atf_space* s, uint64_t first_lo, uint64_t first_hi, int64_t n,
                                      int64_t* d_out, int64_t ld, void* stream) {
  return decode128_common(s, nullptr, nullptr, first_lo, first_hi, n, d_out, ld, stream, true);
}

atf_status atf_space_value_bits(const atf_space* s, int32_t* bits) {
  if (!s || !bits) return ATF_ERR_INVALID_ARG;
  *bits = space_v64(s) ? 64 : 32;
  return ATF_OK;
}

atf_status atf_space_stats(const atf_space* s, atf_level_stats* out, int32_t cap, int32_t* n_out) {
  if (!s || !n_out) return ATF_ERR_INVALID_ARG;
  if (s->state < GENERATED) return ATF_ERR_STATE;
  int n = 0;
  for (size_t g = 0; g < s->groups.size(); g++)
    for (size_t k = 0; k < s->groups[g].levels.size(); k++) {
      if (out && n < cap) {
        const LevelPlan& lp = s->groups[g].levels[k];
        const LevelData& d = s->data[g][k];
        atf_level_stats& o = out[n];
        o.group = (int32_t)g;
        o.level = (int32_t)k;
        o.param = lp.param;
        o.r = lp.r;
        o.evals = d.evals;
        o.f = d.n;
        o.ms = d.ms;
        o.path = lp.generic ? 1 : 0;
        o.expand_ms = d.expand_ms;
        o.kernel = d.kernel;
        o.pairs = d.pairs;
        o.cpt = d.cpt;
        o.nseg = d.nseg;
        o.launches = d.launches;
      }
      n++;
    }
  *n_out = n;
  return ATF_OK;
}

// ---------------------------------------------------------------- multi-GPU shards
// every rank computes the prefix levels up to the cut k* (first level
// with f >= 1024 * world) and the level k*+1 of the whole cut frontier; rank r then
// keeps the contiguous slice of level-k* nodes whose level-(k*+1) child prefix lies in
// [r T / world, (r+1) T / world) and expands its children locally.  Concatenating the
// ranks' slices in rank order gives the single-GPU arrays.
atf_status atf_space_generate_shard(atf_space* s, int32_t rank, int32_t world, int64_t* h_counts, int32_t cap,
                                    int32_t* n_out) {
  if (!s || !n_out || world < 1 || rank < 0 || rank >= world) return fail(s, ATF_ERR_INVALID_ARG, "bad rank/world");
  if (s->state == BUILDING) {
    atf_status e = atf_space_plan(s);
    if (e) return e;
  }
  if (s->dev_ready && s->ipc_alloc) release_device(s);
  s->ipc_alloc = false;
  s->replay_ok = false;
  drop_graph(s);
  atf_status e = ensure_device(s);
  if (e) return e;
  size_t G = s->groups.size();
  s->data.assign(G, {});
  s->tails.assign(G, {});
  for (size_t g = 0; g < G; g++) {
    s->data[g].assign(s->groups[g].levels.size(), LevelData{});
    for (auto& c : s->arena[g]) c.used = 0;
  }
  s->shard_rank = rank;
  s->shard_world = world;
  s->shard_cut.assign(G, 0);
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  const uint64_t thresh = 1024ull * (uint64_t)world;
  // phase 1: replicated prefix, level by level, until the cut
  std::vector<const uint32_t*> fr(G, s->d_root);
  std::vector<uint64_t> fz(G, 1);
  std::vector<int> kk(G, 0);
  std::vector<char> cut_done(G, 0);
  for (;;) {
    std::vector<int> gs;
    for (size_t g = 0; g < G; g++) {
      int L = (int)s->groups[g].levels.size();
      // expand while the frontier is small, and always the level just after the cut
      if (cut_done[g] || kk[g] >= L) continue;
      gs.push_back((int)g);
    }
    if (gs.empty()) break;
    for (int g : gs) {
      std::vector<int> one{g}, k1{kk[g]};
      std::vector<const uint32_t*> f1{fr[g]};
      std::vector<uint64_t> z1{fz[g]};
      // run exactly one level: temporarily cap the group's level count
      GroupPlan& gp = s->groups[g];
      std::vector<LevelPlan> saved(gp.levels.begin() + kk[g] + 1, gp.levels.end());
      gp.levels.resize(kk[g] + 1);
      e = run_levels(s, one, k1, f1, z1);
      gp.levels.insert(gp.levels.end(), saved.begin(), saved.end());
      if (e) return e;
      LevelData& d = s->data[g][kk[g]];
      fr[g] = d.rec;
      fz[g] = d.n;
      kk[g]++;
      // cut after the level following the first level with >= thresh nodes
      if (kk[g] >= 2 && s->data[g][kk[g] - 2].n >= thresh) cut_done[g] = 2;  // sharded
      else if (d.n == 0) cut_done[g] = 1;                                      // empty: replicated
    }
  }
  // phase 2: slice the cut level (k* = kk-2) by the child counts of level k*+1
  std::vector<int> gs, kf;
  std::vector<const uint32_t*> f2;
  std::vector<uint64_t> z2;
  for (size_t g = 0; g < G; g++) {
    int L = (int)s->groups[g].levels.size();
    if (cut_done[g] != 2) {
      // group too small to shard: fully replicated, owned by rank 0
      s->shard_cut[g] = L;
      continue;
    }
    int kc = kk[g] - 2;  // cut level
    s->shard_cut[g] = kc + 1;
    LevelData& cutd = s->data[g][kc];
    uint64_t ncut = cutd.n;
    std::vector<uint64_t> csr(ncut + 1);
    CUDA_TRY(s, cudaMemcpyAsync(csr.data(), cutd.csr, (ncut + 1) * 8, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(s, cudaStreamSynchronize(st));
    uint64_t lo = 0, hi = 0;
    shard_slice(csr.data(), ncut, rank, world, &lo, &hi);
    // slice of level k*+1 = children of cut nodes [lo, hi)
    LevelData& nd = s->data[g][kc + 1];
    uint64_t c0 = csr[lo], c1 = csr[hi];
    GroupPlan& gp = s->groups[g];
    nd.offset = c0;
    nd.rec = nd.rec + c0 * gp.words;
    nd.n = c1 - c0;
    if (kc + 2 < L) {
      gs.push_back((int)g);
      kf.push_back(kc + 2);
      f2.push_back(nd.rec);
      z2.push_back(nd.n);
    }
  }
  if (!gs.empty()) {
    if ((e = run_levels(s, gs, kf, f2, z2))) return e;
  }
  // counts: per (group, level): this rank's nodes of the sharded levels; replicated levels
  // count on rank 0 only, so that the sum over ranks is the global level size.
  int n = 0;
  for (size_t g = 0; g < G; g++)
    for (size_t k = 0; k < s->groups[g].levels.size(); k++) {
      int64_t c = (int)k >= s->shard_cut[g] ? (int64_t)s->data[g][k].n : (rank == 0 ? (int64_t)s->data[g][k].n : 0);
      if (h_counts && n < cap) h_counts[n] = c;
      n++;
    }
  *n_out = n;
  s->state = SHARDED;
  return ATF_OK;
}

atf_status atf_space_finalize_shard(atf_space* s, const int64_t* all, int32_t world, int32_t n) {
  if (!s || !all) return ATF_ERR_INVALID_ARG;
  if (s->state != SHARDED) return fail(s, ATF_ERR_STATE, "finalize_shard needs generate_shard");
  if (world != s->shard_world) return fail(s, ATF_ERR_INVALID_ARG, "world mismatch");
  int idx = 0;
  size_t G = s->groups.size();
  s->gsize.assign(G, 0);
  cudaStream_t st = (cudaStream_t)s->opts.stream;
  for (size_t g = 0; g < G; g++)
    for (size_t k = 0; k < s->groups[g].levels.size(); k++, idx++) {
      if (idx >= n) return fail(s, ATF_ERR_INVALID_ARG, "counts too short");
      uint64_t before = 0, tot = 0;
      shard_offsets(all, world, n, idx, s->shard_rank, &before, &tot);
      LevelData& d = s->data[g][k];
      if ((int)k >= s->shard_cut[g]) {
        uint64_t old = d.offset;
        d.offset = before;
        // CSR entries of this rank's sharded parents point into its local child array;
        // shift them to global child indices
        if ((int)k > s->shard_cut[g] && k >= 1) {
          LevelData& pdl = s->data[g][k - 1];
          if (pdl.csr && pdl.n) {
            int ce = launch_add_offset(pdl.csr, pdl.n + 1, before, st);
            if (ce) return fail(s, ATF_ERR_CUDA, "csr fix-up");
          }
        }
        (void)old;
      }
      if (k + 1 == s->groups[g].levels.size()) s->gsize[g] = tot;
    }
  s->state = FINAL_SHARD;  // sizes global; decode needs the whole tree (not available)
  return ATF_OK;
}

atf_status atf_test_jit_source(atf_space* s, int32_t g, int32_t k, char* buf, size_t cap, size_t* len_out) {
  if (!s) return ATF_ERR_INVALID_ARG;
  atf_status e = plan(s);
  if (e) return e;
  if (g < 0 || g >= (int)s->groups.size() || k < 0 || k >= (int)s->groups[g].levels.size()) return ATF_ERR_INVALID_ARG;
  const GroupPlan& gp = s->groups[g];
  const LevelPlan& lp = gp.levels[k];
  LevelArgs a = lp.proto;
  a.r = lp.r;
  a.n_parents = 1;
  choose_geometry(a, gp.words, false);
  a.mask_bytes = a.r <= 8 ? 1 : (a.r <= 16 ? 2 : (a.r <= 32 ? 4 : 8));
  const auto& vals = s->params[lp.param].values;
  std::vector<uint32_t> mags(vals.size());
  for (size_t j = 0; j < vals.size(); j++) {
    const uint32_t ax = vals[j] < 0 ? 0u - (uint32_t)vals[j] : (uint32_t)vals[j];
    mags[j] = ax ? 0xffffffffu / ax + 1u : 0x10000u;
  }
  // narrow fast levels: the pass-1 kernel; mid-width nf_ok levels: the exact-mask kernel
  const std::string src = a.kind == K_NFAST ? jit_nfast_source(a, gp.words, vals, mags)
                          : (a.kind == K_WTILE && a.nf_ok && a.r <= kWideJitMax) ? jit_wide_source(a, gp.words, vals, mags)
                                                                                 : std::string();
  if (len_out) *len_out = src.size();
  if (buf && cap) {
    const size_t n = std::min(cap - 1, src.size());
    memcpy(buf, src.data(), n);
    buf[n] = 0;
  }
  return ATF_OK;
}

atf_status atf_space_generate_dist(atf_space* s, int32_t rank, int32_t world, atf_allgather_fn allgather, void* ctx) {
  if (!s || !allgather || world < 1 || rank < 0 || rank >= world) return fail(s, ATF_ERR_INVALID_ARG, "bad rank/world");
  if (s->state == BUILDING) {
    atf_status e = atf_space_plan(s);
    if (e) return e;
  }
  s->replay_ok = false;
  drop_graph(s);
  if (s->dev_ready && !s->ipc_alloc) release_device(s);  // arenas must be exportable (cudaMalloc)
  s->ipc_alloc = true;
  atf_status e = ensure_device(s);
  if (e) return e;
  const size_t G = s->groups.size();
  dist_reset(s);
  if ((s->opts.flags & ATF_FLAG_TIMING) && s->events.size() != G) {
    s->events.assign(G, {});
    for (size_t g = 0; g < G; g++) {
      s->events[g].resize(s->groups[g].levels.size());
      for (auto& ev : s->events[g]) {
        CUDA_TRY(s, cudaEventCreate(&ev.first));
        CUDA_TRY(s, cudaEventCreate(&ev.mid));
        CUDA_TRY(s, cudaEventCreate(&ev.second));
      }
    }
  }
  return generate_dist_impl(s, rank, world, allgather, ctx);
}

atf_status atf_space_dist_round_ms(const atf_space* s, float* out, int32_t cap, int32_t* n_out) {
  if (!s || !n_out || cap < 0) return ATF_ERR_INVALID_ARG;
  if (s->dist_round_ms.empty()) return ATF_ERR_STATE;
  *n_out = (int32_t)s->dist_round_ms.size();
  if (out)
    for (int32_t i = 0; i < cap && i < *n_out; i++) out[i] = s->dist_round_ms[i];
  return ATF_OK;
}

atf_status atf_test_set_geometry(int32_t tiles_per_sm, int32_t repl_log2) {
  if (tiles_per_sm < 0 || tiles_per_sm > 4096 || repl_log2 < 0 || repl_log2 > 62) return ATF_ERR_INVALID_ARG;
  g_tiles_per_sm.store(tiles_per_sm ? tiles_per_sm : 256);
  g_repl_log2.store(repl_log2 ? repl_log2 : 28);
  return ATF_OK;
}

atf_status atf_test_set_direct_tiles(int32_t n) {
  if (n < 0 || n > (1 << 20)) return ATF_ERR_INVALID_ARG;
  g_direct_tiles.store(n ? n : 16);
  return ATF_OK;
}

atf_status atf_test_set_async_rounds(int32_t on) {
  g_async_rounds.store(on ? 1 : 0);
  return ATF_OK;
}

atf_status atf_test_set_wide_group(int32_t n) {
  if (n != 0 && n != 2 && n != 4 && n != 8 && n != 16) return ATF_ERR_INVALID_ARG;
  jit_set_wide_group(n ? n : 4);
  return ATF_OK;
}

atf_status atf_test_set_tail_leaf_direct(int32_t mode) {
  if (mode < 0 || mode > 2) return ATF_ERR_INVALID_ARG;
  jit_set_tail_leaf_direct(mode);
  return ATF_OK;
}

atf_status atf_test_set_tail_product(int32_t on) {
  jit_set_tail_product(on != 0);
  return ATF_OK;
}

atf_status atf_test_set_tail_stage(int32_t bytes) {
  if (bytes != 0 && (bytes < 2048 || bytes > 49152 || bytes % 16)) return ATF_ERR_INVALID_ARG;
  jit_set_tail_stage(bytes);
  return ATF_OK;
}

atf_status atf_test_tail_source(atf_space* s, int32_t g, char* buf, size_t cap, size_t* len_out, int32_t* k0_out) {
  if (!s) return ATF_ERR_INVALID_ARG;
  atf_status e = plan(s);
  if (e) return e;
  if (g < 0 || g >= (int)s->groups.size()) return ATF_ERR_INVALID_ARG;
  const GroupPlan& gp = s->groups[g];
  const int k0 = tail_start(s, g);
  if (k0_out) *k0_out = k0;
  std::string src;
  if (k0 >= 0) {
    const TailArgs t = tail_protos(gp, k0);
    std::vector<std::vector<int32_t>> cx;
    std::vector<std::vector<uint32_t>> cm;
    std::vector<std::vector<int>> pvl;
    tail_jit_inputs(s, gp, k0, t.nl, cx, cm, pvl);
    src = jit_tail_source(t, gp.words, cx, cm, k0, pvl);
  }
  if (len_out) *len_out = src.size();
  if (buf && cap) {
    const size_t n = std::min(cap - 1, src.size());
    memcpy(buf, src.data(), n);
    buf[n] = 0;
  }
  return ATF_OK;
}

atf_status atf_test_divisible16(uint64_t* h_mismatches) {
  if (!h_mismatches) return ATF_ERR_INVALID_ARG;
  unsigned long long* d = nullptr;
  if (cudaMalloc(&d, 8) != cudaSuccess) return ATF_ERR_CUDA;
  cudaMemset(d, 0, 8);
  int ce = launch_divisible16_check(d, nullptr);
  unsigned long long h = ~0ull;
  if (!ce) ce = (int)cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  cudaFree(d);
  *h_mismatches = h;
  return ce ? ATF_ERR_CUDA : ATF_OK;
}

atf_status atf_test_exclusive_scan_u32(const uint32_t* d_in, uint64_t* d_out, int64_t n, void* stream) {
  if ((!d_in && n > 0) || !d_out || n < 0) return ATF_ERR_INVALID_ARG;
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t tiles = n > 0 ? (n + 1023) / 1024 : 1;
  unsigned long long* status = nullptr;
  unsigned int* counter = nullptr;
  if (cudaMallocAsync((void**)&status, tiles * 8, st) != cudaSuccess) return ATF_ERR_OOM;
  if (cudaMallocAsync((void**)&counter, 4, st) != cudaSuccess) return ATF_ERR_OOM;
  cudaMemsetAsync(status, 0, tiles * 8, st);
  cudaMemsetAsync(counter, 0, 4, st);
  if (n == 0) cudaMemsetAsync(d_out, 0, 8, st);
  else if (launch_scan_u32(d_in, d_out, n, status, counter, st)) return ATF_ERR_CUDA;
  cudaFreeAsync(status, st);
  cudaFreeAsync(counter, st);
  return cudaStreamSynchronize(st) == cudaSuccess ? ATF_OK : ATF_ERR_CUDA;
}

atf_status atf_test_shard_slice(const uint64_t* h_csr, uint64_t ncut, int32_t rank, int32_t world, uint64_t* lo,
                                uint64_t* hi) {
  if (!h_csr || !lo || !hi || world < 1 || rank < 0 || rank >= world) return ATF_ERR_INVALID_ARG;
  shard_slice(h_csr, ncut, rank, world, lo, hi);
  return ATF_OK;
}

atf_status atf_test_shard_offsets(const int64_t* h_all, int32_t world, int32_t n, int32_t rank, uint64_t* before,
                                  uint64_t* tot) {
  if (!h_all || !before || !tot || world < 1 || n < 0 || rank < 0 || rank >= world) return ATF_ERR_INVALID_ARG;
  for (int i = 0; i < n; i++) shard_offsets(h_all, world, n, i, rank, before + i, tot + i);
  return ATF_OK;
}

void atf_space_destroy(atf_space* s) {
  if (!s) return;
  if (s->dev_ready) {
    cudaSetDevice(s->opts.device);
    release_device(s);
    cudaStreamSynchronize((cudaStream_t)s->opts.stream);
  }
  delete s;
}

}  // extern "C"
