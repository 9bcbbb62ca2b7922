#include <atomic>
// jit.cpp — level-specialised narrow kernels compiled at plan time with NVRTC for sm_100a.
//
// A narrow fast level (expand_nfast, r <= 32) evaluates the same few conjuncts for every
// frontier node; the generic kernel reads the level program from the parameter bank and
// dispatches per term and per operand.  Here the level program is turned into straight-line
// CUDA: field positions, operand kinds, constants, the r candidate values and their divisor
// magics become immediates, each conjunct a fully unrolled bit loop.  The kernel computes
// exactly what expand_nfast pass 1 computes (per-parent accept mask + warp-tile child
// counts; nfast_emit and the scan are shared).  NVRTC is loaded with dlopen; if it is absent
// or a compile fails, the generic kernel runs (still on the GPU).  Compiled kernels are
// cached per source text for the life of the process.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "atf_internal.hpp"

namespace atf {
namespace {

typedef int nvrtcResult_;
typedef struct _nvrtcProgram* nvrtcProgram_;
struct Nvrtc {
  bool ok = false;
  nvrtcResult_ (*create)(nvrtcProgram_*, const char*, const char*, int, const char* const*, const char* const*);
  nvrtcResult_ (*compile)(nvrtcProgram_, int, const char* const*);
  nvrtcResult_ (*cubin_size)(nvrtcProgram_, size_t*);
  nvrtcResult_ (*cubin)(nvrtcProgram_, char*);
  nvrtcResult_ (*log_size)(nvrtcProgram_, size_t*);
  nvrtcResult_ (*log)(nvrtcProgram_, char*);
  nvrtcResult_ (*destroy)(nvrtcProgram_*);
};

Nvrtc& nvrtc() {
  static Nvrtc n;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* names[] = {"libnvrtc.so.12", "libnvrtc.so", "/usr/local/cuda/lib64/libnvrtc.so.12"};
    void* h = nullptr;
    for (const char* nm : names)
      if ((h = dlopen(nm, RTLD_NOW | RTLD_LOCAL))) break;
    if (!h) return;
    n.create = (decltype(n.create))dlsym(h, "nvrtcCreateProgram");
    n.compile = (decltype(n.compile))dlsym(h, "nvrtcCompileProgram");
    n.cubin_size = (decltype(n.cubin_size))dlsym(h, "nvrtcGetCUBINSize");
    n.cubin = (decltype(n.cubin))dlsym(h, "nvrtcGetCUBIN");
    n.log_size = (decltype(n.log_size))dlsym(h, "nvrtcGetProgramLogSize");
    n.log = (decltype(n.log))dlsym(h, "nvrtcGetProgramLog");
    n.destroy = (decltype(n.destroy))dlsym(h, "nvrtcDestroyProgram");
    n.ok = n.create && n.compile && n.cubin_size && n.cubin && n.destroy;
  });
  return n;
}

// Kernel parameters of the generated kernel (same layout on both sides).
struct JitArgs {
  const uint32_t* parent_rec;
  uint64_t n_parents, n_tiles;
  void* masks;
  uint32_t* tile_total;
  const int32_t* pv_range[kMaxSlots];
  const uint32_t* pv_magic[kMaxSlots];
};

const char* kPrelude = R"(
typedef unsigned int u32; typedef unsigned long long u64; typedef int i32; typedef long long i64;
struct JitArgs { const u32* parent_rec; u64 n_parents, n_tiles; void* masks; u32* tile_total;
                 const i32* pv_range[24]; const u32* pv_magic[24]; };
__device__ __forceinline__ u32 uabs(i64 v) { return (u32)(v < 0 ? -v : v); }
__device__ __forceinline__ bool divisible16(u32 nb, u32 q) {  // as in dev_common.cuh
  float rq;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(rq) : "f"((float)q));
  const u32 k = __float2uint_rn((float)nb * rq);
  return k * q == nb;
}
)";

std::string hex(uint32_t v) {
  char b[16];
  snprintf(b, sizeof b, "0x%xu", v);
  return b;
}

// Source of the level kernel, or "" if the level uses something the generator does not
// cover (then the generic kernel runs).
std::string gen_source(const LevelArgs& a, int W, const std::vector<int32_t>& cx, const std::vector<uint32_t>& cm) {
  if (a.kind != K_NFAST || a.n_terms == 0 || a.r > 64 || (int)cx.size() != a.r) return "";
  const int r = a.r;
  const bool wide = r > 32;  // 64-bit masks
  const std::string MT = wide ? "u64" : "u32";
  std::string s = kPrelude;
  s += "extern \"C\" __global__ void __launch_bounds__(256) atf_nfast_jit(const __grid_constant__ JitArgs a) {\n";
  s += "  const int lane = threadIdx.x & 31;\n";
  s += "  const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;\n";
  s += "  for (u64 t = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5; t < a.n_tiles; t += nw) {\n";
  s += "    u32 cnt = 0;\n";
  // all parent records of the lane first (vector loads, independent), then the nodes
  const std::string NPL = std::to_string(kNfNPL), TNs = std::to_string(32 * kNfNPL), Ws = std::to_string(W);
  s += "    u32 rq[" + NPL + "][" + Ws + "];\n";
  s += "#pragma unroll\n    for (int q = 0; q < " + NPL + "; q++) {\n";
  s += "      const u64 nd = t * " + TNs + "ull + (u64)q * 32 + lane;\n";
  if (a.level == 0) {
    s += "      for (int w = 0; w < " + Ws + "; w++) rq[q][w] = 0u;\n";
  } else {
    s += "      if (nd < a.n_parents) {\n";
    if (W == 1) s += "        rq[q][0] = __ldg(a.parent_rec + nd);\n";
    else if (W == 2) s += "        const uint2 v = __ldg(reinterpret_cast<const uint2*>(a.parent_rec) + nd);\n"
                          "        rq[q][0] = v.x; rq[q][1] = v.y;\n";
    else
      for (int h = 0; h < W / 4; h++)
        s += "        { const uint4 v = __ldg(reinterpret_cast<const uint4*>(a.parent_rec) + nd * " + std::to_string(W / 4) +
             " + " + std::to_string(h) + "); rq[q][" + std::to_string(4 * h) + "] = v.x; rq[q][" + std::to_string(4 * h + 1) +
             "] = v.y; rq[q][" + std::to_string(4 * h + 2) + "] = v.z; rq[q][" + std::to_string(4 * h + 3) + "] = v.w; }\n";
    s += "      }\n";
  }
  s += "    }\n";
  s += "#pragma unroll\n    for (int q = 0; q < " + NPL + "; q++) {\n";
  s += "      const u64 nd = t * " + TNs + "ull + (u64)q * 32 + lane;\n";
  s += "      if (nd >= a.n_parents) continue;\n";
  for (int w = 0; w < W; w++) s += "      const u32 w" + std::to_string(w) + " = rq[q][" + std::to_string(w) + "];\n";
  // ancestor values (and magics) used by the terms
  std::vector<int> need_v(a.n_pv, 0), need_m(a.n_pv, 0);
  auto mark = [&](const NfOp& o, bool mag) {
    if (o.kind == NF_PV) { need_v[o.s1] = 1; if (mag) need_m[o.s1] = 1; }
    if (o.kind == NF_PROD) { need_v[o.s1] = 1; need_v[o.s2] = 1; }
  };
  for (int t = 0; t < a.n_terms; t++) {
    const Term& T = a.terms[t];
    mark(a.nf_op[t][0], T.kind == T_MULX || T.kind == T_DIVPROD);
    if (T.kind == T_DIVPROD || T.kind == T_QDIV || T.kind == T_CMP) mark(a.nf_op[t][1], false);
  }
  for (int p = 0; p < a.n_pv; p++) {
    if (!need_v[p]) continue;
    const std::string ps = std::to_string(p);
    const uint32_t bits = (uint32_t)a.pv_bits[p];
    std::string pos = bits ? "((w" + std::to_string(a.pv_word[p]) + " >> " + std::to_string(a.pv_shift[p]) + ") & " +
                                 hex(bits >= 32 ? 0xffffffffu : ((1u << bits) - 1u)) + ")"
                           : std::string("0u");
    s += "      const u32 p" + ps + " = " + pos + ";\n";
    s += "      const i64 v" + ps + " = (i64)__ldg(a.pv_range[" + ps + "] + p" + ps + ");\n";
    if (need_m[p]) s += "      const u32 g" + ps + " = __ldg(a.pv_magic[" + ps + "] + p" + ps + ");\n";
  }
  auto sval = [&](const NfOp& o) -> std::string {
    if (o.kind == NF_CONST) return "(i64)" + std::to_string(o.c) + "ll";
    if (o.kind == NF_PV) return "v" + std::to_string(o.s1);
    return "(v" + std::to_string(o.s1) + " * v" + std::to_string(o.s2) + ")";
  };
  auto magic = [&](const NfOp& o, const std::string& absname) -> std::string {
    if (o.kind == NF_CONST) return hex(o.cm);
    if (o.kind == NF_PV) return "(" + absname + " == 0u ? 0u : g" + std::to_string(o.s1) + ")";
    return "(" + absname + " > 1u ? 0xffffffffu / " + absname + " + 1u : 0u)";
  };
  const unsigned long long full = r >= 64 ? ~0ull : ((1ull << r) - 1ull);
  char fb[32];
  snprintf(fb, sizeof fb, "0x%llxull", full);
  s += "      " + MT + " m = (" + MT + ")" + fb + ";\n";
  for (int t = 0; t < a.n_terms; t++) {
    const Term& T = a.terms[t];
    const NfOp& oa = a.nf_op[t][0];
    const NfOp& ob = a.nf_op[t][1];
    const std::string ts = std::to_string(t);
    s += "      if (m) {  // term " + ts + "\n";
    auto divx_bits = [&](const std::string& n) {
      std::string b = "        " + MT + " mm = 0u;\n";
      for (int c = 0; c < r; c++)
        if (cx[c] != 0) b += "        mm |= (" + MT + ")(" + n + " * " + hex(cm[c]) + " < 0x10000u) << " + std::to_string(c) + ";\n";
      b += "        m &= mm;\n";
      return b;
    };
    switch (T.kind) {
      case T_DIVX:
        s += "        const u32 n" + ts + " = uabs(" + sval(oa) + ");\n" + divx_bits("n" + ts);
        break;
      case T_DIVPROD:
        s += "        const u32 av = uabs(" + sval(oa) + "), bv = uabs(" + sval(ob) + ");\n";
        s += "        const u32 ma = " + magic(oa, "av") + ";\n";
        s += "        const u32 n" + ts + " = av == 1u ? bv : __umulhi(bv, ma);\n";
        s += "        if (av == 0u || n" + ts + " * av != bv) m = 0u;\n";
        s += "        else {\n" + divx_bits("n" + ts) + "        }\n";
        break;
      case T_MULX: {
        s += "        const u32 d = uabs(" + sval(oa) + ");\n";
        s += "        const u32 md = " + magic(oa, "d") + ", md1 = md - 1u;\n";
        s += "        if (d == 0u) m = 0u;\n        else {\n          " + MT + " mm = 0u;\n";
        for (int c = 0; c < r; c++) {
          const uint32_t ax = cx[c] < 0 ? 0u - (uint32_t)cx[c] : (uint32_t)cx[c];
          s += "          mm |= (" + MT + ")(" + hex(ax) + " * md <= md1) << " + std::to_string(c) + ";\n";
        }
        s += "          m &= mm;\n        }\n";
        break;
      }
      case T_QDIV: {
        s += "        const u32 num = uabs(" + sval(oa) + "), nb = uabs(" + sval(ob) + ");\n";
        s += "        " + MT + " mm = 0u;\n";
        for (int c = 0; c < r; c++) {
          const uint32_t ax = cx[c] < 0 ? 0u - (uint32_t)cx[c] : (uint32_t)cx[c];
          if (ax == 0) continue;  // x == 0 rejects
          const std::string q = ax == 1 ? std::string("num") : "__umulhi(num, " + hex(cm[c]) + ")";
          s += "        if ((m >> " + std::to_string(c) + ") & 1u) { const u32 q = " + q +
               "; if (q != 0u && divisible16(nb, q)) mm |= (" + MT + ")1u << " + std::to_string(c) + "; }\n";
        }
        s += "        m &= mm;\n";
        break;
      }
      case T_CMP: {
        static const char* rel[] = {"==", "!=", "<", "<=", ">", ">="};
        if (T.rel < R_EQ || T.rel > R_GE) return "";
        s += "        const i32 A = (i32)" + sval(oa) + ", B = (i32)" + sval(ob) + ";\n        " + MT + " mm = 0u;\n";
        for (int c = 0; c < r; c++)
          s += "        mm |= (" + MT + ")(A * " + std::to_string(cx[c]) + " " + rel[T.rel - R_EQ] + " B) << " +
               std::to_string(c) + ";\n";
        s += "        m &= mm;\n";
        break;
      }
      default: return "";
    }
    s += "      }\n";
  }
  // x == 0 candidates get no bit in the DIVX / DIVPROD / QDIV loops
  s += "      cnt += __popcll((u64)m);\n";
  const char* mt = a.mask_bytes == 1 ? "unsigned char" : (a.mask_bytes == 2 ? "unsigned short" : (a.mask_bytes == 4 ? "u32" : "u64"));
  s += std::string("      reinterpret_cast<") + mt + "*>(a.masks)[nd] = (" + mt + ")m;\n";
  s += "    }\n";
  s += "#pragma unroll\n    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);\n";
  s += "    if (lane == 0) a.tile_total[t] = cnt;\n  }\n}\n";
  return s;
}

// ---------------------------------------------------------------- fused narrow tail
// Operand code of level program `a` over a record held in w[] (field positions as immediates,
// ancestor values / magics from the level's tables `tab`).  `pfx` makes the names unique.
struct OpGen {
  const LevelArgs& a;
  std::string tab, pfx;
  std::vector<int> need_v, need_m;
  OpGen(const LevelArgs& a_, std::string tab_, std::string pfx_)
      : a(a_), tab(std::move(tab_)), pfx(std::move(pfx_)), need_v(a_.n_pv, 0), need_m(a_.n_pv, 0) {}
  void mark(const NfOp& o, bool mag) {
    if (o.kind == NF_PV) { need_v[o.s1] = 1; if (mag) need_m[o.s1] = 1; }
    if (o.kind == NF_PROD) { need_v[o.s1] = 1; need_v[o.s2] = 1; }
  }
  void mark_term(int t) {
    const Term& T = a.terms[t];
    mark(a.nf_op[t][0], T.kind == T_MULX || T.kind == T_DIVPROD);
    if (T.kind == T_DIVPROD || T.kind == T_QDIV || T.kind == T_CMP) mark(a.nf_op[t][1], false);
  }
  std::string loads(const std::string& ind) const {  // value (and magic) loads of the marked slots
    std::string s;
    for (int p = 0; p < a.n_pv; p++) {
      if (!need_v[p]) continue;
      const std::string ps = std::to_string(p), nm = pfx + ps;
      const uint32_t bits = (uint32_t)a.pv_bits[p];
      std::string pos = bits ? "((w[" + std::to_string(a.pv_word[p]) + "] >> " + std::to_string(a.pv_shift[p]) + ") & " +
                                   hex(bits >= 32 ? 0xffffffffu : ((1u << bits) - 1u)) + ")"
                             : std::string("0u");
      s += ind + "const u32 p" + nm + " = " + pos + ";\n";
      s += ind + "const i64 v" + nm + " = (i64)__ldg(a." + tab + "_range[" + ps + "] + p" + nm + ");\n";
      if (need_m[p]) s += ind + "const u32 g" + nm + " = __ldg(a." + tab + "_magic[" + ps + "] + p" + nm + ");\n";
    }
    return s;
  }
  std::string sval(const NfOp& o) const {
    if (o.kind == NF_CONST) return "(i64)" + std::to_string(o.c) + "ll";
    if (o.kind == NF_PV) return "v" + pfx + std::to_string(o.s1);
    return "(v" + pfx + std::to_string(o.s1) + " * v" + pfx + std::to_string(o.s2) + ")";
  }
  std::string magic(const NfOp& o, const std::string& absname) const {
    if (o.kind == NF_CONST) return hex(o.cm);
    if (o.kind == NF_PV) return "(" + absname + " == 0u ? 0u : g" + pfx + std::to_string(o.s1) + ")";
    return "(" + absname + " > 1u ? 0xffffffffu / " + absname + " + 1u : 0u)";
  }
};

// Per-term node operands -> u32 words (a term's "node constants"): DIVX n | DIVPROD n, or
// 0xffffffff when the gate a | b fails | MULX md, md - 1, d == 0 | QDIV num, nb | CMP A, B.
int nc_words(const Term& T) { return T.kind == T_MULX ? 3 : (T.kind == T_QDIV || T.kind == T_CMP) ? 2 : 1; }
std::string nc_code(const LevelArgs& a, int t, const OpGen& g, const std::string& dst, const std::string& ind) {
  const Term& T = a.terms[t];
  const NfOp& oa = a.nf_op[t][0];
  const NfOp& ob = a.nf_op[t][1];
  std::string s = ind + "{\n";
  switch (T.kind) {
    case T_DIVX: s += ind + "  " + dst + "[0] = uabs(" + g.sval(oa) + ");\n"; break;
    case T_DIVPROD:
      s += ind + "  const u32 av = uabs(" + g.sval(oa) + "), bv = uabs(" + g.sval(ob) + ");\n";
      s += ind + "  const u32 ma = " + g.magic(oa, "av") + ";\n";
      s += ind + "  const u32 n = av == 1u ? bv : __umulhi(bv, ma);\n";
      s += ind + "  " + dst + "[0] = (av == 0u || n * av != bv) ? 0xffffffffu : n;\n";
      break;
    case T_MULX:
      s += ind + "  const u32 d = uabs(" + g.sval(oa) + ");\n";
      s += ind + "  const u32 md = " + g.magic(oa, "d") + ";\n";
      s += ind + "  " + dst + "[0] = md; " + dst + "[1] = md - 1u; " + dst + "[2] = d == 0u;\n";
      break;
    case T_QDIV:
      s += ind + "  " + dst + "[0] = uabs(" + g.sval(oa) + "); " + dst + "[1] = uabs(" + g.sval(ob) + ");\n";
      break;
    default:
      s += ind + "  " + dst + "[0] = (u32)(i32)" + g.sval(oa) + "; " + dst + "[1] = (u32)(i32)" + g.sval(ob) + ";\n";
  }
  return s + ind + "}\n";
}

// Mask code of term t from its node constants `nc` (base index i0) over r <= 64 candidates
// (mask type u32 for r <= 32, else u64).
std::string term_mask_code(const LevelArgs& a, int t, const std::vector<int32_t>& cx, const std::vector<uint32_t>& cm,
                           const std::string& nc) {
  const Term& T = a.terms[t];
  const int r = a.r;
  const std::string MT = r > 32 ? "u64" : "u32";
  std::string s = "  if (m) {  // term " + std::to_string(t) + "\n    " + MT + " mm = 0u;\n";
  switch (T.kind) {
    case T_DIVX: case T_DIVPROD:
      s += "    const u32 n = " + nc + "[0];\n";
      if (T.kind == T_DIVPROD) s += "    if (n == 0xffffffffu) m = 0u;\n";
      for (int c = 0; c < r; c++)
        if (cx[c] != 0) s += "    mm |= (" + MT + ")(n * " + hex(cm[c]) + " < 0x10000u) << " + std::to_string(c) + ";\n";
      break;
    case T_MULX:
      s += "    const u32 md = " + nc + "[0], mq = " + nc + "[1];\n    if (" + nc + "[2]) m = 0u;\n";
      for (int c = 0; c < r; c++) {
        const uint32_t ax = cx[c] < 0 ? 0u - (uint32_t)cx[c] : (uint32_t)cx[c];
        s += "    mm |= (" + MT + ")(" + hex(ax) + " * md <= mq) << " + std::to_string(c) + ";\n";
      }
      break;
    case T_QDIV:
      s += "    const u32 num = " + nc + "[0], nb = " + nc + "[1];\n";
      for (int c = 0; c < r; c++) {
        const uint32_t ax = cx[c] < 0 ? 0u - (uint32_t)cx[c] : (uint32_t)cx[c];
        if (ax == 0) continue;  // x == 0 rejects
        const std::string q = ax == 1 ? std::string("num") : "__umulhi(num, " + hex(cm[c]) + ")";
        s += "    if ((m >> " + std::to_string(c) + ") & 1u) { const u32 q = " + q +
             "; if (q != 0u && divisible16(nb, q)) mm |= (" + MT + ")1u << " + std::to_string(c) + "; }\n";
      }
      break;
    default: {
      static const char* rel[] = {"==", "!=", "<", "<=", ">", ">="};
      s += "    const i32 A = (i32)" + nc + "[0], B = (i32)" + nc + "[1];\n";
      for (int c = 0; c < r; c++)
        s += "    mm |= (" + MT + ")(A * " + std::to_string(cx[c]) + " " + rel[T.rel - R_EQ] + " B) << " + std::to_string(c) + ";\n";
    }
  }
  return s + "    m &= mm;\n  }\n";
}

// Kernel parameters of the generated tail kernels (same layout on both sides).
struct TailJitArgs {
  const uint32_t* parent_rec;
  uint64_t n_parents, n_tiles;
  uint32_t* tile_total;
  const uint64_t* tile_base;
  uint32_t* node_cnt;  // [nl][n_parents] subtree counts per frontier node (count -> emit)
  uint64_t* csr[kMaxTail];
  uint32_t* rec[kMaxTail];
  const int32_t* l0_range[kMaxSlots];
  const uint32_t* l0_magic[kMaxSlots];
  const int32_t* l1_range[kMaxSlots];
  const uint32_t* l1_magic[kMaxSlots];
  const int32_t* l2_range[kMaxSlots];
  const uint32_t* l2_magic[kMaxSlots];
  const int32_t* l3_range[kMaxSlots];
  const uint32_t* l3_magic[kMaxSlots];
};

const char* kTailPrelude = R"(
struct TailJitArgs { const u32* parent_rec; u64 n_parents, n_tiles; u32* tile_total; const u64* tile_base;
                     u32* node_cnt; u64* csr[4]; u32* rec[4];
                     const i32* l0_range[24]; const u32* l0_magic[24]; const i32* l1_range[24]; const u32* l1_magic[24];
                     const i32* l2_range[24]; const u32* l2_magic[24]; const i32* l3_range[24]; const u32* l3_magic[24]; };
)";

// Source of the two tail kernels for levels lv[0..nl) (group levels k0..k0+nl-1; pv_level[d][s] =
// the group level of slot s's ancestor).  A term whose operands all come from levels above the
// tail ("node constants") is evaluated ONCE per frontier node (tnc) instead of once per tail node:
// every tail node below a frontier node shares those ancestors.
//   atf_tail_count: thread per frontier node, depth-first subtree counts (node constants in
//                   registers), warp-tile totals per level.
//   atf_tail_emit:  warp tile = 32 frontier nodes; every tail level in chunks of 32 nodes in
//                   canonical order; children staged in per-warp shared-memory buffers (with the
//                   frontier lane they descend from, whose node constants sit in shared memory),
//                   written out as coalesced vectors, CSR entries of every chunk.
// tail emit staging bytes per warp (atf_test_set_tail_stage); 0 = by the tail: 12 KB when its first
// level has more than 32 candidates (C3-IS4 1.59 -> 1.54 ms), else 8 KB (C3-IS2: 6 KB 1.72, 8 KB 1.69,
// 12 KB 1.75 ms; profiles/r02_tail_stage_sweep.txt)
std::atomic<int> g_tail_stage{0};
std::atomic<bool> g_tail_product{true};  // product-structured tails (atf_test_set_tail_product)
// leaf pass writes global memory instead of the staging area: 0 never, 1 always, 2 (default) when the
// tail's first level has more than 32 candidates (u64 masks: C3-IS4 1.62 -> 1.58 ms; C3-IS2, r = 25,
// measured 1.69 -> 1.77 ms the other way; tools/tail_leaf_ab.py)
std::atomic<int> g_tail_leaf_direct{2};
std::atomic<int> g_wide_group{4};  // atf_wide_jit: candidates per superset group (atf_test_set_wide_group)

std::string gen_tail_source(const TailArgs& t, int W, const std::vector<std::vector<int32_t>>& cx,
                            const std::vector<std::vector<uint32_t>>& cm, int k0,
                            const std::vector<std::vector<int>>& pv_level, int* warp_bytes, bool* product_out = nullptr) {
  const int nl = t.nl;
  if (nl < 2 || nl > kMaxTail || (int)pv_level.size() < nl) return "";
  std::string s = kPrelude;
  s += kTailPrelude;
  const std::string Ws = std::to_string(W);
  // node-constant layout: (level, term) -> first word; hoisted iff every operand is above the tail
  std::vector<std::vector<int>> ncoff(nl);
  int NNC = 0;
  for (int d = 0; d < nl; d++) {
    const LevelArgs& a = t.lv[d];
    // masks: u32, or u64 for 32 < r <= 64 on a non-leaf level (the leaf masks are staged as u32)
    if (a.n_terms == 0 || a.r > (d + 1 < nl ? 64 : 32) || a.r < 1 || (int)cx[d].size() != a.r) return "";
    auto above = [&](const NfOp& o) {
      if (o.kind == NF_CONST) return true;
      if (o.kind == NF_PV) return pv_level[d][o.s1] < k0;
      return pv_level[d][o.s1] < k0 && pv_level[d][o.s2] < k0;
    };
    ncoff[d].assign(a.n_terms, -1);
    for (int tt = 0; tt < a.n_terms; tt++) {
      const Term& T = a.terms[tt];
      if (T.kind == T_CMP && (T.rel < R_EQ || T.rel > R_GE)) return "";
      if (T.kind != T_DIVX && T.kind != T_DIVPROD && T.kind != T_MULX && T.kind != T_QDIV && T.kind != T_CMP) return "";
      const bool two = T.kind == T_DIVPROD || T.kind == T_QDIV || T.kind == T_CMP;
      if (above(a.nf_op[tt][0]) && (!two || above(a.nf_op[tt][1]))) {
        ncoff[d][tt] = NNC;
        NNC += nc_words(T);
      }
    }
  }
  const int NC = std::max(NNC, 1);
  // tnc: node constants of a frontier node
  s += "__device__ __forceinline__ void tnc(const TailJitArgs& a, const u32* w, u32* nc) {\n";
  for (int d = 0; d < nl; d++) {
    OpGen g(t.lv[d], "l" + std::to_string(d), std::to_string(d) + "_");
    for (int tt = 0; tt < t.lv[d].n_terms; tt++)
      if (ncoff[d][tt] >= 0) g.mark_term(tt);
    s += "  {\n" + g.loads("    ");
    for (int tt = 0; tt < t.lv[d].n_terms; tt++)
      if (ncoff[d][tt] >= 0) s += nc_code(t.lv[d], tt, g, "(nc + " + std::to_string(ncoff[d][tt]) + ")", "    ");
    s += "  }\n";
  }
  s += "}\n";
  // tmask_d(w, nc): hoisted terms from nc, the others from the node's own record
  for (int d = 0; d < nl; d++) {
    const LevelArgs& a = t.lv[d];
    OpGen g(a, "l" + std::to_string(d), "");
    for (int tt = 0; tt < a.n_terms; tt++)
      if (ncoff[d][tt] < 0) g.mark_term(tt);
    const std::string MT = a.r > 32 ? "u64" : "u32";
    s += "__device__ __forceinline__ " + MT + " tmask" + std::to_string(d) + "(const TailJitArgs& a, const u32* w, const u32* nc) {\n";
    s += g.loads("  ");
    if (a.r > 32)
      s += "  u64 m = " + (a.r == 64 ? std::string("0xffffffffffffffffull") : "((1ull << " + std::to_string(a.r) + ") - 1ull)") + ";\n";
    else
      s += "  u32 m = " + hex(a.r >= 32 ? 0xffffffffu : ((1u << a.r) - 1u)) + ";\n";
    for (int tt = 0; tt < a.n_terms; tt++) {
      if (ncoff[d][tt] >= 0) {
        s += term_mask_code(a, tt, cx[d], cm[d], "(nc + " + std::to_string(ncoff[d][tt]) + ")");
      } else {
        s += "  {\n    u32 lc[3];\n" + nc_code(a, tt, g, "lc", "    ");
        s += term_mask_code(a, tt, cx[d], cm[d], "lc") + "  }\n";
      }
    }
    s += "  return m;\n}\n";
  }
  // ---- product-structured count: every term of every tail level reads only ancestors above the
  // tail (all node constants), so under one frontier node level d's mask m_d is the same at every
  // level-(d-1) node and level d holds P_d = c_0 ... c_d nodes (c_e = popc m_e): the count is a
  // product instead of a depth-first walk (C3-IS2 145 -> 108 us).  The emit stays the depth-first
  // kernel below (a lane-parallel emit over the product grid was built and measured slower: 0.97 vs
  // 0.69 ms).
  bool product = g_tail_product.load();
  for (int d = 0; d < nl && product; d++)
    for (int tt = 0; tt < t.lv[d].n_terms; tt++)
      if (ncoff[d][tt] < 0) product = false;
  if (product_out) *product_out = product;
  if (product) {
    const std::string NLs = std::to_string(nl);
    // count: thread per frontier node
    s += "extern \"C\" __global__ void __launch_bounds__(256) atf_tail_count(const __grid_constant__ TailJitArgs a) {\n";
    s += "  const int lane = threadIdx.x & 31;\n  const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;\n";
    s += "  for (u64 tile = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5; tile < a.n_tiles; tile += nw) {\n";
    s += "    const u64 nd = tile * 32 + lane;\n    u32 P[" + NLs + "] = {};\n";
    s += "    if (nd < a.n_parents) {\n      u32 w[" + Ws + "];\n";
    s += "      for (int i = 0; i < " + Ws + "; i++) w[i] = __ldg(a.parent_rec + nd * " + Ws + " + i);\n";
    s += "      u32 nc[" + std::to_string(NC) + "];\n      tnc(a, w, nc);\n      u32 p = 1u;\n";
    for (int d = 0; d < nl; d++)
      s += "      p *= (u32)__popcll((u64)tmask" + std::to_string(d) + "(a, w, nc)); P[" + std::to_string(d) + "] = p;\n";
    for (int d = 0; d < nl; d++)
      s += "      a.node_cnt[(u64)" + std::to_string(d) + " * a.n_parents + nd] = P[" + std::to_string(d) + "];\n";
    s += "    }\n";
    for (int d = 0; d < nl; d++) {
      const std::string ds = std::to_string(d);
      s += "    { u32 v = P[" + ds + "];\n#pragma unroll\n      for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);\n";
      s += "      if (lane == 0) a.tile_total[(u64)" + ds + " * a.n_tiles + tile] = v; }\n";
    }
    s += "  }\n}\n";
  }
  auto child = [&](int d, const std::string& src, const std::string& dst, const std::string& ind) {
    std::string c;
    const int fw = t.lv[d].field_word, fs = t.lv[d].field_shift;
    for (int w = 0; w < W; w++)
      c += ind + dst + "[" + std::to_string(w) + "] = " + src + "[" + std::to_string(w) + "]" +
           (w == fw && t.lv[d].r > 1 ? " | (cc << " + std::to_string(fs) + ")" : "") + ";\n";  // r == 1: no field bits
    return c;
  };
  if (!product) {  // (the product count above replaces it)
    // ---- count: depth-first per frontier node
    for (int d = nl - 1; d >= 0; d--) {
      const std::string ds = std::to_string(d);
      s += "__device__ __forceinline__ void cnt" + ds + "(const TailJitArgs& a, const u32* w, const u32* nc, u32* cnt) {\n";
      s += "  auto m = tmask" + ds + "(a, w, nc);\n  cnt[" + ds + "] += __popcll((u64)m);\n";
      if (d + 1 < nl) {
        s += "  while (m) {\n    const u32 cc = __ffsll((long long)m) - 1;\n    m &= m - 1;\n    u32 cw[" + Ws + "];\n";
        s += child(d, "w", "cw", "    ");
        s += "    cnt" + std::to_string(d + 1) + "(a, cw, nc, cnt);\n  }\n";
      }
      s += "}\n";
    }
    s += "extern \"C\" __global__ void __launch_bounds__(256) atf_tail_count(const __grid_constant__ TailJitArgs a) {\n";
    s += "  const int lane = threadIdx.x & 31;\n  const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;\n";
    s += "  for (u64 tile = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5; tile < a.n_tiles; tile += nw) {\n";
    s += "    const u64 nd = tile * 32 + lane;\n    u32 cnt[" + std::to_string(nl) + "] = {};\n";
    s += "    if (nd < a.n_parents) {\n      u32 w[" + Ws + "];\n";
    s += "      for (int i = 0; i < " + Ws + "; i++) w[i] = __ldg(a.parent_rec + nd * " + Ws + " + i);\n";
    s += "      u32 nc[" + std::to_string(NC) + "];\n      tnc(a, w, nc);\n      cnt0(a, w, nc, cnt);\n";
    for (int d = 0; d < nl; d++)
      s += "      a.node_cnt[(u64)" + std::to_string(d) + " * a.n_parents + nd] = cnt[" + std::to_string(d) + "];\n";
    s += "    }\n";
    for (int d = 0; d < nl; d++) {
      const std::string ds = std::to_string(d);
      s += "    { u32 v = cnt[" + ds + "];\n#pragma unroll\n      for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);\n";
      s += "      if (lane == 0) a.tile_total[(u64)" + ds + " * a.n_tiles + tile] = v; }\n";
    }
    s += "  }\n}\n";
  }
  // ---- emit: lane = frontier node, depth-first (like the count), output staged per warp.
  // Each lane recounts its subtree (cnt_d); warp scans give its nodes' tile-local positions per
  // level (a node's level-d descendants come out of a depth-first walk in canonical order).  The
  // warp then writes the tile in "parts": runs of consecutive lanes whose output (records, and
  // CSR entries as u32 offsets from the child level's tile base) fits the warp's staging area;
  // the lanes of a part write their subtrees into shared memory, the warp copies every level's
  // run out as coalesced words.  A single lane whose subtree alone exceeds the area writes
  // straight to global memory.
  const int kStage = g_tail_stage.load() > 0 ? g_tail_stage.load() : (t.lv[0].r > 32 ? 12288 : 8192);  // per warp
  if (warp_bytes) *warp_bytes = kStage;
  const std::string NLs = std::to_string(nl), NCs = std::to_string(NC), RB = std::to_string(W * 4);
  // The leaf level is not written by the depth-first walk when staged: a level-(nl-2) node stores
  // its leaf mask instead (and advances the leaf cursor by its popcount), and a balanced pass over
  // the part's level-(nl-2) nodes (lane-strided) writes the leaves afterwards, so the walk's
  // divergence does not reach the largest level.
  const int LP = nl - 2;  // parents of the leaves
  for (int d = nl - 1; d >= 0; d--) {
    const std::string ds = std::to_string(d);
    s += "__device__ __forceinline__ void dfs" + ds + "(const TailJitArgs& a, const u32* w, const u32* nc, u32* cur, "
         "const u64* base, const u32* pb, unsigned char* sm, bool staged, const u32* roff, const u32* coff, u32 lmo) {\n";
    s += "  auto m = tmask" + ds + "(a, w, nc);\n";
    s += "  while (m) {\n    const u32 cc = __ffsll((long long)m) - 1;\n    m &= m - 1;\n    u32 cw[" + Ws + "];\n";
    s += child(d, "w", "cw", "    ");
    s += "    const u32 slot = cur[" + ds + "]++;\n";
    s += "    if (staged) {\n      u32* dst = reinterpret_cast<u32*>(sm + roff[" + ds + "]) + (slot - pb[" + ds + "]) * " + Ws + ";\n";
    for (int w = 0; w < W; w++) s += "      dst[" + std::to_string(w) + "] = cw[" + std::to_string(w) + "];\n";
    s += "    } else {\n      u32* dst = a.rec[" + ds + "] + (base[" + ds + "] + slot) * " + Ws + ";\n";
    for (int w = 0; w < W; w++) s += "      dst[" + std::to_string(w) + "] = cw[" + std::to_string(w) + "];\n";
    s += "    }\n";
    if (d + 1 < nl) {
      const std::string d1 = std::to_string(d + 1);
      s += "    if (staged) reinterpret_cast<u32*>(sm + coff[" + ds + "])[slot - pb[" + ds + "]] = cur[" + d1 + "];\n";
      s += "    else a.csr[" + d1 + "][base[" + ds + "] + slot] = base[" + d1 + "] + cur[" + d1 + "];\n";
      if (d == LP) {
        s += "    if (staged) {\n      const u32 lm = tmask" + d1 + "(a, cw, nc);\n";
        s += "      reinterpret_cast<u32*>(sm + lmo)[slot - pb[" + ds + "]] = lm;\n      cur[" + d1 + "] += __popc(lm);\n";
        s += "    } else {\n      dfs" + d1 + "(a, cw, nc, cur, base, pb, sm, staged, roff, coff, lmo);\n    }\n";
      } else {
        s += "    dfs" + d1 + "(a, cw, nc, cur, base, pb, sm, staged, roff, coff, lmo);\n";
      }
    }
    s += "  }\n}\n";
  }
  s += "extern \"C\" __global__ void __launch_bounds__(128) atf_tail_emit(const __grid_constant__ TailJitArgs a) {\n";
  s += "  extern __shared__ __align__(16) unsigned char smem[];\n";
  s += "  const int lane = threadIdx.x & 31;\n  unsigned char* sm = smem + (threadIdx.x >> 5) * " + std::to_string(kStage) + ";\n";
  s += "  const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;\n  const u64 gw = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;\n";
  s += "  if (gw == 0 && lane < " + NLs + ") {\n";
  s += "    const u64 above = lane == 0 ? a.n_parents : a.tile_base[(u64)(lane - 1) * (a.n_tiles + 1) + a.n_tiles];\n";
  s += "    a.csr[lane][above] = a.tile_base[(u64)lane * (a.n_tiles + 1) + a.n_tiles];\n  }\n";
  // the next tile's parent records, subtree counts and tile bases are loaded while this tile is
  // emitted (software pipelining over the persistent grid-stride loop)
  auto load_next = [&](const std::string& t, const std::string& ind) {
    std::string c;
    c += ind + "{ const u64 xn = " + t + " * 32 + lane; const bool xv = xn < a.n_parents;\n";
    c += ind + "  for (int i = 0; i < " + Ws + "; i++) pw_[i] = xv ? __ldg(a.parent_rec + xn * " + Ws + " + i) : 0u;\n";
    for (int d = 0; d < nl; d++)
      c += ind + "  pc_[" + std::to_string(d) + "] = xv ? __ldcs(a.node_cnt + (u64)" + std::to_string(d) + " * a.n_parents + xn) : 0u;\n";
    for (int d = 0; d < nl; d++)
      c += ind + "  pb_[" + std::to_string(d) + "] = a.tile_base[(u64)" + std::to_string(d) + " * (a.n_tiles + 1) + " + t + "];\n";
    c += ind + "}\n";
    return c;
  };
  s += "  u32 pw_[" + Ws + "], pc_[" + NLs + "];\n  u64 pb_[" + NLs + "];\n";
  s += "  if (gw < a.n_tiles) {\n" + load_next("gw", "    ") + "  }\n";
  s += "  for (u64 tile = gw; tile < a.n_tiles; tile += nw) {\n";
  s += "    const u64 nd = tile * 32 + lane;\n    const bool valid = nd < a.n_parents;\n    u32 w[" + Ws + "], cnt[" + NLs + "];\n    u64 base[" + NLs + "];\n";
  s += "#pragma unroll\n    for (int i = 0; i < " + Ws + "; i++) w[i] = pw_[i];\n";
  s += "#pragma unroll\n    for (int d = 0; d < " + NLs + "; d++) { cnt[d] = pc_[d]; base[d] = pb_[d]; }\n";
  s += "    if (tile + nw < a.n_tiles) {\n" + load_next("(tile + nw)", "      ") + "    }\n";
  s += "    u32 nc[" + NCs + "];\n";
  s += "    if (valid) tnc(a, w, nc);\n";
  s += "    u32 off[" + NLs + "];\n    u32 bytes = 0;\n";
  s += "#pragma unroll\n    for (int d = 0; d < " + NLs + "; d++) {\n";
  s += "      u32 incl = cnt[d];\n#pragma unroll\n      for (int o = 1; o < 32; o <<= 1) { const u32 y = __shfl_up_sync(0xffffffffu, incl, o); "
       "if (lane >= o) incl += y; }\n";
  s += "      off[d] = incl - cnt[d];\n";
  const int ldm = g_tail_leaf_direct.load();  // leaves straight to global memory (no staging)?
  const bool leaf_direct = ldm == 1 || (ldm == 2 && t.lv[0].r > 32);
  s += "      bytes += cnt[d] * (" + (leaf_direct ? "(d + 1 < " + NLs + " ? " + RB + "u : 0u)" : RB + "u") + " + (d + 1 < " + NLs +
       " ? 4u : 0u) + (d == " + std::to_string(nl - 2) + " ? 4u : 0u));\n    }\n";
  s += "    if (valid) a.csr[0][nd] = base[0] + off[0];\n";
  // inclusive byte prefix per lane
  s += "    u32 bincl = bytes;\n#pragma unroll\n    for (int o = 1; o < 32; o <<= 1) { const u32 y = __shfl_up_sync(0xffffffffu, bincl, o); "
       "if (lane >= o) bincl += y; }\n";
  s += "    for (int p0 = 0; p0 < 32;) {\n";
  s += "      const u32 b0 = p0 ? __shfl_sync(0xffffffffu, bincl, p0 - 1) : 0u;\n";
  s += "      const unsigned fit = __ballot_sync(0xffffffffu, lane >= p0 && bincl - b0 <= " + std::to_string(kStage - 16) + "u);  // 16: the record region's alignment\n";
  s += "      const int p1 = fit ? 32 - __clz(fit) : p0 + 1;  // lanes [p0, p1)\n";
  s += "      const bool staged = fit != 0u;\n";
  s += "      u32 pb[" + NLs + "], pe[" + NLs + "], roff[" + NLs + "], coff[" + NLs + "];\n";
  s += "      u32 o = 0;\n";
  s += "#pragma unroll\n      for (int d = 0; d < " + NLs + "; d++) {\n";
  s += "        pb[d] = __shfl_sync(0xffffffffu, off[d], p0);\n";
  s += "        const u32 last = __shfl_sync(0xffffffffu, off[d] + cnt[d], p1 - 1);\n        pe[d] = last;\n";
  s += "        if (d + 1 < " + NLs + ") { coff[d] = o; o += (last - pb[d]) * 4u; }\n      }\n";
  s += "      const u32 lmo = o;  // leaf masks of the part's level-" + std::to_string(nl - 2) + " nodes\n";
  s += "      o += (pe[" + std::to_string(nl - 2) + "] - pb[" + std::to_string(nl - 2) + "]) * 4u;\n";
  s += "      o = (o + 15u) & ~15u;\n";
  s += "#pragma unroll\n      for (int d = 0; d < " + NLs + "; d++) { roff[d] = o; o += " +
       (leaf_direct ? "(d + 1 < " + NLs + " ? (pe[d] - pb[d]) * " + RB + "u : 0u)" : "(pe[d] - pb[d]) * " + RB + "u") + "; }\n";
  s += "      if (lane >= p0 && lane < p1 && valid) {\n        u32 cur[" + NLs + "];\n";
  s += "#pragma unroll\n        for (int d = 0; d < " + NLs + "; d++) cur[d] = off[d];\n";
  s += "        dfs0(a, w, nc, cur, base, pb, sm, staged, roff, coff, lmo);\n      }\n";
  s += "      if (staged) {\n        __syncwarp();\n";
  {  // balanced leaf pass
    const std::string lp = std::to_string(nl - 2), ll = std::to_string(nl - 1);
    const int fw = t.lv[nl - 1].field_word, fs = t.lv[nl - 1].field_shift;
    s += "        {  // leaves of the part's level-" + lp + " nodes, lane-strided\n";
    s += "          const u32 nn = pe[" + lp + "] - pb[" + lp + "];\n";
    s += "          const u32* lms = reinterpret_cast<const u32*>(sm + lmo);\n";
    s += "          const u32* cst = reinterpret_cast<const u32*>(sm + coff[" + lp + "]);\n";
    s += "          for (u32 i = lane; i < nn; i += 32) {\n            u32 lm = lms[i];\n            if (!lm) continue;\n";
    s += "            u32 k = cst[i] - pb[" + ll + "];\n";
    s += "            const u32* pr = reinterpret_cast<const u32*>(sm + roff[" + lp + "]) + i * " + Ws + ";\n";
    s += "            u32 pw[" + Ws + "];\n";
    for (int w = 0; w < W; w++) s += "            pw[" + std::to_string(w) + "] = pr[" + std::to_string(w) + "];\n";
    s += "            while (lm) {\n              const u32 cc = __ffs(lm) - 1;\n              lm &= lm - 1;\n";
    if (leaf_direct)
      s += "              u32* dst = a.rec[" + ll + "] + (base[" + ll + "] + pb[" + ll + "] + k) * " + Ws + ";\n";
    else
      s += "              u32* dst = reinterpret_cast<u32*>(sm + roff[" + ll + "]) + k * " + Ws + ";\n";
    for (int w = 0; w < W; w++)
      s += "              dst[" + std::to_string(w) + "] = pw[" + std::to_string(w) + "]" +
           (w == fw && t.lv[nl - 1].r > 1 ? " | (cc << " + std::to_string(fs) + ")" : "") + ";\n";
    s += "              k++;\n            }\n          }\n          __syncwarp();\n        }\n";
  }
  s += "#pragma unroll\n        for (int d = 0; d < " + NLs + "; d++) {\n";
  s += "          const u32 n = " + (leaf_direct ? "d + 1 < " + NLs + " ? (pe[d] - pb[d]) * " + Ws + "u : 0u" : "(pe[d] - pb[d]) * " + Ws + "u") + ";\n";
  s += "          const u32* src = reinterpret_cast<const u32*>(sm + roff[d]);\n          u32* dst = a.rec[d] + (base[d] + pb[d]) * " + Ws + ";\n";
  if (W % 2 == 0)  // 8-byte aligned on both sides (records of even W, 8-byte CSR regions before them)
    s += "          { const uint2* s2 = reinterpret_cast<const uint2*>(src); uint2* d2 = reinterpret_cast<uint2*>(dst);\n"
         "#pragma unroll 4\n            for (u32 v = lane; v < n / 2; v += 32) d2[v] = s2[v]; }\n";
  else
    s += "#pragma unroll 4\n          for (u32 v = lane; v < n; v += 32) dst[v] = src[v];\n";
  s += "          if (d + 1 < " + NLs + ") {\n            const u32* cs = reinterpret_cast<const u32*>(sm + coff[d]);\n";
  s += "            u64* cd = a.csr[d + 1] + base[d] + pb[d];\n            const u64 cb = base[d + 1 < " + NLs + " ? d + 1 : d];\n";
  s += "#pragma unroll 4\n            for (u32 v = lane; v < pe[d] - pb[d]; v += 32) cd[v] = cb + cs[v];\n          }\n";
  s += "        }\n        __syncwarp();\n      }\n      p0 = p1;\n    }\n  }\n}\n";
  return s;
}


// ---------------------------------------------------------------- mid-width levels
// A narrow-fast-style level (nf_ok: every conjunct an atom over ancestor values / constants /
// ancestor products) with 32 < r <= kWideJitMax candidates: lane = frontier node, the
// candidates in words of 32.  Per word, the first conjunct (the cheapest, host order) is
// evaluated EXACTLY for every candidate with the candidate's magic / |value| as an immediate
// (one IMAD + compare per pair, no item recomputation as in the warp-tile kernel's
// superset filter); the other conjuncts run only on that word's survivors (table loads).
// The per-node word masks stay in the warp's shared memory for the emit.  Output protocol =
// expand_wtile's stash path (tile = 32 nodes: tile_total / tile_seg / stash segment claimed
// by atomicAdd, tile-local CSR), so scan_kernel + level_emit_kernel finish the level.
struct WideJitArgs {
  const uint32_t* parent_rec;
  uint64_t n_parents, n_tiles;
  const int32_t* pv_range[kMaxSlots];
  const uint32_t* pv_magic[kMaxSlots];
  const int32_t* cand;
  const uint32_t* cand_magic;
  const uint32_t* cand_abs;
  uint64_t* csr;
  uint32_t* stash;
  uint64_t stash_cap;
  unsigned long long* stash_top;
  uint32_t* tile_total;
  unsigned long long* tile_seg;
  unsigned int* overflow_flag;
};

const char* kWidePrelude = R"(
struct WideJitArgs { const u32* parent_rec; u64 n_parents, n_tiles; const i32* pv_range[24]; const u32* pv_magic[24];
                     const i32* cand; const u32* cand_magic; const u32* cand_abs; u64* csr; u32* stash; u64 stash_cap;
                     u64* stash_top; u32* tile_total; u64* tile_seg; u32* overflow_flag; };
)";

constexpr int kWideStageWords = 1024;  // u32 words of records staged per warp for coalesced stash writes

std::string gen_wide_source(const LevelArgs& a, int W, const std::vector<int32_t>& cx, const std::vector<uint32_t>& cm) {
  const int r = a.r;
  if (!a.nf_ok || r <= 32 || r > kWideJitMax || (int)cx.size() != r || a.n_gates) return "";
  const int NWD = (r + 31) / 32;
  const std::string Ws = std::to_string(W);
  std::string s = kPrelude;
  s += kWidePrelude;
  const int stage = kWideStageWords / W;           // records
  const int stride = NWD * 32 + kWideStageWords;   // u32 per warp
  s += "extern \"C\" __global__ void __launch_bounds__(256) atf_wide_jit(const __grid_constant__ WideJitArgs a) {\n";
  s += "  extern __shared__ __align__(16) u32 smem[];\n  const int lane = threadIdx.x & 31;\n";
  s += "  u32* s_m = smem + (threadIdx.x >> 5) * " + std::to_string(stride) + ";\n";
  s += "  u32* s_st = s_m + " + std::to_string(NWD * 32) + ";\n";
  s += "  const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;\n";
  s += "  for (u64 tile = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5; tile < a.n_tiles; tile += nw) {\n";
  s += "    const u64 nd = tile * 32 + lane;\n    const bool valid = nd < a.n_parents;\n    u32 w[" + Ws + "];\n";
  if (a.level == 0) s += "    for (int i = 0; i < " + Ws + "; i++) w[i] = 0u;\n";
  else s += "    for (int i = 0; i < " + Ws + "; i++) w[i] = valid ? __ldg(a.parent_rec + nd * " + Ws + " + i) : 0u;\n";
  // operands
  std::vector<int> need_v(a.n_pv, 0), need_m(a.n_pv, 0);
  auto mark = [&](const NfOp& o, bool mag) {
    if (o.kind == NF_PV) { need_v[o.s1] = 1; if (mag) need_m[o.s1] = 1; }
    if (o.kind == NF_PROD) { need_v[o.s1] = 1; need_v[o.s2] = 1; }
  };
  for (int t = 0; t < a.n_terms; t++) {
    const Term& T = a.terms[t];
    mark(a.nf_op[t][0], T.kind == T_MULX || T.kind == T_DIVPROD);
    if (T.kind == T_DIVPROD || T.kind == T_QDIV || T.kind == T_CMP) mark(a.nf_op[t][1], false);
  }
  for (int p = 0; p < a.n_pv; p++) {
    if (!need_v[p]) continue;
    const std::string ps = std::to_string(p);
    const uint32_t bits = (uint32_t)a.pv_bits[p];
    std::string pos = bits ? "((w[" + std::to_string(a.pv_word[p]) + "] >> " + std::to_string(a.pv_shift[p]) + ") & " +
                                 hex(bits >= 32 ? 0xffffffffu : ((1u << bits) - 1u)) + ")"
                           : std::string("0u");
    s += "    const u32 p" + ps + " = " + pos + ";\n";
    s += "    const i64 v" + ps + " = (i64)__ldg(a.pv_range[" + ps + "] + p" + ps + ");\n";
    if (need_m[p]) s += "    const u32 g" + ps + " = __ldg(a.pv_magic[" + ps + "] + p" + ps + ");\n";
  }
  auto sval = [&](const NfOp& o) -> std::string {
    if (o.kind == NF_CONST) return "(i64)" + std::to_string(o.c) + "ll";
    if (o.kind == NF_PV) return "v" + std::to_string(o.s1);
    return "(v" + std::to_string(o.s1) + " * v" + std::to_string(o.s2) + ")";
  };
  auto magic = [&](const NfOp& o, const std::string& absname) -> std::string {
    if (o.kind == NF_CONST) return hex(o.cm);
    if (o.kind == NF_PV) return "(" + absname + " == 0u ? 0u : g" + std::to_string(o.s1) + ")";
    return "(" + absname + " > 1u ? 0xffffffffu / " + absname + " + 1u : 0u)";
  };
  // per-term node operands (and node gate from DIVPROD / MULX: the node accepts nothing)
  s += "    bool alive = valid;\n";
  for (int t = 0; t < a.n_terms; t++) {
    const Term& T = a.terms[t];
    const NfOp& oa = a.nf_op[t][0];
    const NfOp& ob = a.nf_op[t][1];
    const std::string ts = std::to_string(t);
    switch (T.kind) {
      case T_DIVX: s += "    const u32 n" + ts + " = uabs(" + sval(oa) + ");\n"; break;
      case T_DIVPROD:
        s += "    u32 n" + ts + ";\n    { const u32 av = uabs(" + sval(oa) + "), bv = uabs(" + sval(ob) + ");\n";
        s += "      const u32 ma = " + magic(oa, "av") + ";\n";
        s += "      n" + ts + " = av == 1u ? bv : __umulhi(bv, ma);\n";
        s += "      if (av == 0u || n" + ts + " * av != bv) alive = false; }\n";
        break;
      case T_MULX:
        s += "    const u32 d" + ts + " = uabs(" + sval(oa) + ");\n";
        s += "    const u32 md" + ts + " = " + magic(oa, "d" + ts) + ", mq" + ts + " = md" + ts + " - 1u;\n";
        s += "    if (d" + ts + " == 0u) alive = false;\n";
        break;
      case T_QDIV:
        s += "    const u32 num" + ts + " = uabs(" + sval(oa) + "), nb" + ts + " = uabs(" + sval(ob) + ");\n";
        break;
      case T_CMP:
        if (T.rel < R_EQ || T.rel > R_GE) return "";
        s += "    const i32 A" + ts + " = (i32)" + sval(oa) + ", B" + ts + " = (i32)" + sval(ob) + ";\n";
        break;
      default: return "";
    }
  }
  static const char* rel[] = {"==", "!=", "<", "<=", ">", ">="};
  if (a.n_terms > 0 && a.terms[0].kind == T_QDIV) return "";  // a quotient test is never the cheapest conjunct
  s += "    u32 cnt = 0, nzw = 0;  // nzw bit j: candidate word j has survivors\n";
  // first conjunct: divisibility tests (x | n, d | x) in groups of 4 candidates, a superset
  // test per group (min of the 4 magic products, VIMNMX3) whose survivors are re-tested exactly
  // below; comparisons exactly per candidate
  const bool grouped = a.n_terms > 0 && (a.terms[0].kind == T_DIVX || a.terms[0].kind == T_DIVPROD ||
                                         a.terms[0].kind == T_MULX);
  for (int j = 0; j < NWD; j++) {
    s += "    {  // candidates " + std::to_string(32 * j) + ".." + std::to_string(std::min(r, 32 * j + 32) - 1) + "\n";
    s += "      u32 mw = 0u;\n";
    if (grouped) {
      const bool mulx = a.terms[0].kind == T_MULX;
      const int GS = g_wide_group.load();  // candidates per superset group (4; test hook)
      for (int c0 = 0; c0 < 32 && 32 * j + c0 < r; c0 += GS) {
        const int nc = std::min(GS, r - (32 * j + c0));
        std::vector<std::string> pr;
        for (int c = c0; c < c0 + nc; c++) {
          const int ci = 32 * j + c;
          const uint32_t ax = cx[ci] < 0 ? 0u - (uint32_t)cx[ci] : (uint32_t)cx[ci];
          pr.push_back(mulx ? hex(ax) + " * md0" : "n0 * " + hex(cm[ci]));
        }
        while (pr.size() > 1) {  // balanced min tree
          std::vector<std::string> nx;
          for (size_t i = 0; i + 1 < pr.size(); i += 2) nx.push_back("min(" + pr[i] + ", " + pr[i + 1] + ")");
          if (pr.size() % 2) nx.push_back(pr.back());
          pr.swap(nx);
        }
        const std::string q = pr[0];
        s += "      { const u32 q = " + q + "; if (q " + (mulx ? "<= mq0" : "< 0x10000u") + ") mw |= " +
             hex(((1u << nc) - 1u) << c0) + "; }\n";
      }
    } else {
      for (int c = 0; c < 32 && 32 * j + c < r; c++) {
        const int ci = 32 * j + c;
        const std::string sh = " << " + std::to_string(c) + ";\n";
        if (a.n_terms == 0) { s += "      mw |= 1u" + sh; continue; }
        const Term& T = a.terms[0];
        s += "      mw |= (u32)(A0 * " + std::to_string(cx[ci]) + " " + rel[T.rel - R_EQ] + " B0)" + sh;
      }
    }
    if (grouped || a.n_terms > 1) {
      s += "      u32 sv = mw;\n      while (sv) {\n        const int c = __ffs(sv) - 1;\n        sv &= sv - 1;\n";
      s += "        const int ci = " + std::to_string(32 * j) + " + c;\n        bool ok = true;\n";
      for (int t = grouped ? 0 : 1; t < a.n_terms; t++) {
        const Term& T = a.terms[t];
        const std::string ts = std::to_string(t);
        switch (T.kind) {
          case T_DIVX: case T_DIVPROD:
            s += "        { const u32 mg = __ldg(a.cand_magic + ci); ok = ok && mg != 0x10000u && n" + ts + " * mg < 0x10000u; }\n";
            break;
          case T_MULX: s += "        ok = ok && __ldg(a.cand_abs + ci) * md" + ts + " <= mq" + ts + ";\n"; break;
          case T_QDIV:
            s += "        if (ok) { const u32 ax = __ldg(a.cand_abs + ci);\n";
            s += "          const u32 q = ax == 1u ? num" + ts + " : __umulhi(num" + ts + ", __ldg(a.cand_magic + ci));\n";
            s += "          ok = ax != 0u && q != 0u && divisible16(nb" + ts + ", q); }\n";
            break;
          default:
            s += "        ok = ok && (A" + ts + " * __ldg(a.cand + ci) " + rel[T.rel - R_EQ] + " B" + ts + ");\n";
        }
      }
      s += "        if (!ok) mw &= ~(1u << c);\n      }\n";
    }
    s += "      if (!alive) mw = 0u;\n      s_m[" + std::to_string(32 * j) + " + lane] = mw;\n      cnt += __popc(mw);\n";
    s += "      nzw |= (u32)(mw != 0u) << " + std::to_string(j) + ";\n    }\n";
  }
  // tile scan, stash segment, CSR
  s += "    u32 incl = cnt;\n#pragma unroll\n    for (int o = 1; o < 32; o <<= 1) { const u32 y = __shfl_up_sync(0xffffffffu, incl, o); if (lane >= o) incl += y; }\n";
  s += "    const u32 total = __shfl_sync(0xffffffffu, incl, 31);\n    u32 k = incl - cnt;\n";
  s += "    u64 sgb = 0;\n    if (lane == 0) {\n      sgb = total ? atomicAdd(a.stash_top, (u64)total) : 0ull;\n";
  s += "      if (total && sgb + total > a.stash_cap) atomicOr(a.overflow_flag, 1u);\n";
  s += "      a.tile_total[tile] = total;\n      a.tile_seg[tile] = sgb;\n    }\n";
  s += "    sgb = __shfl_sync(0xffffffffu, sgb, 0);\n    if (valid) a.csr[nd] = k;\n";
  s += "    const bool staged = total <= " + std::to_string(stage) + "u;\n";
  s += "    __syncwarp();\n";
  const int fw = a.field_word, fs = a.field_shift;
  s += "    while (nzw) {  // the node's nonzero words only\n      const int j = __ffs(nzw) - 1;\n      nzw &= nzw - 1;\n"
       "      u32 mw = s_m[j * 32 + lane];\n";
  s += "      while (mw) {\n        const u32 c = __ffs(mw) - 1;\n        mw &= mw - 1;\n        const u32 pos = (u32)j * 32u + c;\n";
  s += "        if (staged) {\n";
  for (int wd = 0; wd < W; wd++)
    s += "          s_st[k * " + Ws + " + " + std::to_string(wd) + "] = w[" + std::to_string(wd) + "]" +
         (wd == fw && r > 1 ? " | (pos << " + std::to_string(fs) + ")" : "") + ";\n";
  s += "        } else if (sgb + k < a.stash_cap) {\n";
  for (int wd = 0; wd < W; wd++)
    s += "          a.stash[(sgb + k) * " + Ws + " + " + std::to_string(wd) + "] = w[" + std::to_string(wd) + "]" +
         (wd == fw && r > 1 ? " | (pos << " + std::to_string(fs) + ")" : "") + ";\n";
  s += "        }\n        k++;\n      }\n    }\n";
  s += "    if (staged && sgb + total <= a.stash_cap) {\n      __syncwarp();\n";
  s += "      for (u32 v = lane; v < total * " + Ws + "u; v += 32) a.stash[sgb * " + Ws + " + v] = s_st[v];\n    }\n";
  s += "    __syncwarp();\n  }\n}\n";
  return s;
}

// ---------------------------------------------------------------- batched decode
// The decoder of one generated space (A9): group sizes and their multiply-high
// magics, record widths, field positions and output columns as immediates, so an index costs
// its mixed-radix digits (multiply-high + at most two corrections per group), one leaf gather
// per group (ld.global.cg: 32-byte sectors from L2, no 128-byte L1 line fills for a random
// 8-byte read) and one table load + store per parameter.
struct DecodeJitArgs {
  const uint64_t* idx;
  const uint64_t* digits;
  int64_t n;
  int32_t* out;
  int64_t ld;
  unsigned int* bad;
  const uint32_t* leaves[kMaxGroups];
  const int32_t* range[kMaxLevels];
};

std::string gen_decode_source(const DecodeArgs& a) {
  std::string s = kPrelude;
  s += "struct DecodeJitArgs { const u64* idx; const u64* digits; i64 n; i32* out; i64 ld; u32* bad; "
       "const u32* leaves[" + std::to_string(kMaxGroups) + "]; const i32* range[" + std::to_string(kMaxLevels) + "]; };\n";
  s += "__device__ __forceinline__ uint2 ldcg2(const u32* p) { uint2 v; asm volatile(\"ld.global.cg.v2.u32 {%0,%1}, [%2];\" "
       ": \"=r\"(v.x), \"=r\"(v.y) : \"l\"(p)); return v; }\n";
  s += "__device__ __forceinline__ uint4 ldcg4(const u32* p) { uint4 v; asm volatile(\"ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];\" "
       ": \"=r\"(v.x), \"=r\"(v.y), \"=r\"(v.z), \"=r\"(v.w) : \"l\"(p)); return v; }\n";
  s += "__device__ __forceinline__ u32 ldcg1(const u32* p) { u32 v; asm volatile(\"ld.global.cg.u32 %0, [%1];\" : \"=r\"(v) : \"l\"(p)); return v; }\n";
  unsigned __int128 S = 1;
  bool fits = true;
  for (int g = 0; g < a.n_groups; g++) {
    S *= a.gsize[g];
    if (S >> 64) fits = false;
  }
  char buf[64];
  s += "extern \"C\" __global__ void __launch_bounds__(256) atf_decode_jit(const __grid_constant__ DecodeJitArgs a) {\n";
  s += "  for (i64 i = (i64)blockIdx.x * blockDim.x + threadIdx.x; i < a.n; i += (i64)gridDim.x * blockDim.x) {\n";
  s += "    bool valid = true;\n";
  for (int g = 0; g < a.n_groups; g++) s += "    u64 d" + std::to_string(g) + ";\n";
  s += "    if (a.idx) {\n      u64 rem = __ldcs(a.idx + i);\n";
  snprintf(buf, sizeof buf, "0x%llxull", (unsigned long long)(uint64_t)S);
  s += fits ? "      valid = rem < " + std::string(buf) + ";\n" : "      valid = false;\n";
  for (int g = a.n_groups - 1; g >= 0; g--) {
    const std::string gs = std::to_string(g);
    char sz[32], mg[32];
    snprintf(sz, sizeof sz, "0x%llxull", (unsigned long long)a.gsize[g]);
    snprintf(mg, sizeof mg, "0x%llxull", (unsigned long long)a.gmagic[g]);
    if (a.gsize[g] == 1) { s += "      d" + gs + " = 0;\n"; continue; }
    if (a.gsize[g] == 0) { s += "      d" + gs + " = 0;\n"; continue; }
    s += "      { u64 q = __umul64hi(rem, " + std::string(mg) + "); u64 r = rem - q * " + sz + ";\n";
    s += "        if (r >= " + std::string(sz) + ") { q++; r -= " + sz + "; }\n";
    s += "        if (r >= " + std::string(sz) + ") { q++; r -= " + sz + "; }\n";
    s += "        d" + gs + " = r; rem = q; }\n";
  }
  s += "    } else {\n";
  for (int g = 0; g < a.n_groups; g++) {
    const std::string gs = std::to_string(g);
    char sz[32];
    snprintf(sz, sizeof sz, "0x%llxull", (unsigned long long)a.gsize[g]);
    s += "      d" + gs + " = __ldcs(a.digits + (i64)" + gs + " * a.n + i); valid = valid && d" + gs + " < " + sz + ";\n";
  }
  s += "    }\n";
  s += "    if (!valid) {\n      for (int p = 0; p < " + std::to_string(a.n_params) +
       "; p++) a.out[(i64)p * a.ld + i] = (i32)0x80000000;\n      atomicOr(a.bad, 1u);\n      continue;\n    }\n";
  for (int g = 0; g < a.n_groups; g++) {
    const std::string gs = std::to_string(g);
    const int W = a.words[g];
    s += "    {\n      const u32* rp = a.leaves[" + gs + "] + d" + gs + " * " + std::to_string(W) + "ull;\n";
    if (W == 1) s += "      const u32 w0 = ldcg1(rp);\n";
    else if (W == 2) s += "      const uint2 v = ldcg2(rp); const u32 w0 = v.x, w1 = v.y;\n";
    else {
      s += "      const uint4 v = ldcg4(rp); const u32 w0 = v.x, w1 = v.y, w2 = v.z, w3 = v.w;\n";
      if (W == 8) s += "      const uint4 u = ldcg4(rp + 4); const u32 w4 = u.x, w5 = u.y, w6 = u.z, w7 = u.w;\n";
    }
    for (int l = a.lvl_begin[g]; l < a.lvl_begin[g + 1]; l++) {
      const uint32_t bits = (uint32_t)a.lvl_bits[l];
      std::string pos = bits ? "((w" + std::to_string(a.lvl_word[l]) + " >> " + std::to_string(a.lvl_shift[l]) + ") & " +
                                   hex(bits >= 32 ? 0xffffffffu : ((1u << bits) - 1u)) + ")"
                             : std::string("0u");
      s += "      a.out[(i64)" + std::to_string(a.lvl_param[l]) + " * a.ld + i] = __ldg(a.range[" + std::to_string(l) + "] + " +
           pos + ");\n";
    }
    s += "    }\n";
  }
  s += "  }\n}\n";
  return s;
}

std::mutex g_mu;
std::unordered_map<std::string, cudaLibrary_t> g_cache;  // source -> library (nullptr: failed)

cudaLibrary_t compile_lib(const std::string& src) {
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_cache.find(src);
    if (it != g_cache.end()) return it->second;
  }
  Nvrtc& nv = nvrtc();
  cudaLibrary_t lib = nullptr;
  if (nv.ok) {
    nvrtcProgram_ prog = nullptr;
    if (nv.create(&prog, src.c_str(), "atf_level.cu", 0, nullptr, nullptr) == 0) {
      const char* opts[] = {"-arch=sm_100a", "-std=c++17", "-default-device", "-lineinfo"};
      if (nv.compile(prog, 4, opts) == 0) {
        size_t n = 0;
        nv.cubin_size(prog, &n);
        std::vector<char> cubin(n);
        nv.cubin(prog, cubin.data());
        if (cudaLibraryLoadData(&lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0) != cudaSuccess)
          lib = nullptr;
        cudaGetLastError();
      } else if (nv.log_size && nv.log) {
        size_t n = 0;
        nv.log_size(prog, &n);
        std::string log(n, '\0');
        nv.log(prog, &log[0]);
        fprintf(stderr, "atfgen jit: compile failed (generic kernel used):\n%s\n", log.c_str());
      }
      nv.destroy(&prog);
    }
  }
  std::lock_guard<std::mutex> lk(g_mu);
  g_cache[src] = lib;
  return lib;
}

cudaKernel_t compile(const std::string& src, const char* name = "atf_nfast_jit") {
  cudaLibrary_t lib = compile_lib(src);
  cudaKernel_t k = nullptr;
  if (lib && cudaLibraryGetKernel(&k, lib, name) != cudaSuccess) k = nullptr;
  cudaGetLastError();
  return k;
}

struct TailJit {
  cudaKernel_t count = nullptr, emit = nullptr;
  int warp_bytes = 0, per_sm = 0, per_sm_count = 0;
  bool product = false;  // the count kernel is the product-structured one
};
std::unordered_map<std::string, TailJit> g_tails;  // source -> kernels (under g_mu)

}  // namespace

// Source text of the level's specialised kernel ("" if the level is not covered).
std::string jit_nfast_source(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                             const std::vector<uint32_t>& cand_magics) {
  return gen_source(a, words, cand_values, cand_magics);
}

// Compile (or fetch) the level's specialised pass-1 kernel.  Returns an opaque handle or
// nullptr (the caller then uses the generic kernel).
void* jit_nfast_kernel(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                       const std::vector<uint32_t>& cand_magics) {
  const std::string src = gen_source(a, words, cand_values, cand_magics);
  if (src.empty()) return nullptr;
  return (void*)compile(src);
}

int jit_nfast_launch(void* kernel, const LevelArgs& a, void* stream) {
  JitArgs j;
  std::memset(&j, 0, sizeof j);
  j.parent_rec = a.parent_rec;
  j.n_parents = a.n_parents;
  j.n_tiles = a.n_tiles;
  j.masks = a.masks;
  j.tile_total = a.tile_total;
  for (int i = 0; i < a.n_pv; i++) {
    j.pv_range[i] = a.pv_range[i];
    j.pv_magic[i] = a.pv_magic[i];
  }
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  uint64_t grid = (uint64_t)sms * 8;
  const uint64_t need = (a.n_tiles + 7) / 8;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  void* args[] = {&j};
  cudaError_t e = cudaLaunchKernel((const void*)kernel, dim3((unsigned)grid), dim3(256), args, 0, (cudaStream_t)stream);
  return (int)e;
}


// ---- fused narrow tail: specialised count + emit kernels (nullptr: use the generic ones)
std::string jit_tail_source(const TailArgs& t, int words, const std::vector<std::vector<int32_t>>& cand_values,
                            const std::vector<std::vector<uint32_t>>& cand_magics, int k0,
                            const std::vector<std::vector<int>>& pv_level) {
  return gen_tail_source(t, words, cand_values, cand_magics, k0, pv_level, nullptr);
}

void* jit_tail_kernels(const TailArgs& t, int words, const std::vector<std::vector<int32_t>>& cand_values,
                       const std::vector<std::vector<uint32_t>>& cand_magics, int k0,
                       const std::vector<std::vector<int>>& pv_level) {
  int wb = 0;
  bool prod = false;
  const std::string src = gen_tail_source(t, words, cand_values, cand_magics, k0, pv_level, &wb, &prod);
  if (src.empty()) return nullptr;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_tails.find(src);
    if (it != g_tails.end()) return it->second.count ? (void*)&it->second : nullptr;
  }
  TailJit tj;
  tj.count = compile(src, "atf_tail_count");
  tj.emit = compile(src, "atf_tail_emit");
  tj.warp_bytes = wb;
  tj.product = prod;
  if (tj.count && tj.emit) {
    const int smem = 4 * wb;
    bool ok = !(smem > 48 * 1024 &&
                cudaFuncSetAttribute((const void*)tj.emit, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) !=
                    cudaSuccess);
    int per_sm = 0, per_sm_c = 0;
    if (ok && (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, (const void*)tj.emit, 128, smem) != cudaSuccess ||
               cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm_c, (const void*)tj.count, 256, 0) != cudaSuccess))
      ok = false;
    cudaGetLastError();
    tj.per_sm = per_sm;
    tj.per_sm_count = per_sm_c;
    if (!ok || per_sm < 1 || per_sm_c < 1) tj.count = tj.emit = nullptr;
  } else {
    tj.count = tj.emit = nullptr;
  }
  std::lock_guard<std::mutex> lk(g_mu);
  TailJit& slot = g_tails[src];
  slot = tj;
  return slot.count ? (void*)&slot : nullptr;
}

bool jit_tail_product(void* handle) { return handle && reinterpret_cast<const TailJit*>(handle)->product; }

int jit_tail_launch(void* handle, const TailArgs& t, bool emit, void* stream) {
  const TailJit& tj = *reinterpret_cast<const TailJit*>(handle);
  TailJitArgs j;
  std::memset(&j, 0, sizeof j);
  j.parent_rec = t.parent_rec;
  j.n_parents = t.n_parents;
  j.n_tiles = t.n_tiles;
  j.tile_total = t.tile_total;
  j.tile_base = t.tile_base;
  j.node_cnt = t.node_cnt;
  for (int d = 0; d < kMaxTail; d++) {
    j.csr[d] = t.csr[d];
    j.rec[d] = t.rec[d];
  }
  const int32_t** ranges[4] = {j.l0_range, j.l1_range, j.l2_range, j.l3_range};
  const uint32_t** magics[4] = {j.l0_magic, j.l1_magic, j.l2_magic, j.l3_magic};
  for (int d = 0; d < t.nl; d++)
    for (int i = 0; i < t.lv[d].n_pv; i++) {
      ranges[d][i] = t.lv[d].pv_range[i];
      magics[d][i] = t.lv[d].pv_magic[i];
    }
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  const int threads = emit ? 128 : 256;  // one warp tile (32 frontier nodes) per warp
  uint64_t grid = (uint64_t)sms * (emit ? tj.per_sm : tj.per_sm_count);
  const uint64_t need = (t.n_tiles + threads / 32 - 1) / (threads / 32);
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  void* args[] = {&j};
  cudaError_t e = cudaLaunchKernel((const void*)(emit ? tj.emit : tj.count), dim3((unsigned)grid), dim3(threads), args,
                                   emit ? (size_t)(4 * tj.warp_bytes) : 0, (cudaStream_t)stream);
  return (int)e;
}

// ---- mid-width levels: specialised exact-mask kernel (nullptr: use the warp-tile kernel)
std::string jit_wide_source(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                            const std::vector<uint32_t>& cand_magics) {
  return gen_wide_source(a, words, cand_values, cand_magics);
}

void* jit_wide_kernel(const LevelArgs& a, int words, const std::vector<int32_t>& cand_values,
                      const std::vector<uint32_t>& cand_magics) {
  const std::string src = gen_wide_source(a, words, cand_values, cand_magics);
  if (src.empty()) return nullptr;
  cudaKernel_t k = compile(src, "atf_wide_jit");
  if (!k) return nullptr;
  const int smem = jit_wide_smem(a.r, words);
  if (smem > 48 * 1024 && cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) !=
                              cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return (void*)k;
}

int jit_wide_smem(int r, int words) { (void)words; return 8 * 4 * (((r + 31) / 32) * 32 + kWideStageWords); }

int jit_wide_launch(void* kernel, const LevelArgs& a, int words, void* stream) {
  WideJitArgs j;
  std::memset(&j, 0, sizeof j);
  j.parent_rec = a.parent_rec;
  j.n_parents = a.n_parents;
  j.n_tiles = a.n_tiles;
  for (int i = 0; i < a.n_pv; i++) {
    j.pv_range[i] = a.pv_range[i];
    j.pv_magic[i] = a.pv_magic[i];
  }
  j.cand = a.cand;
  j.cand_magic = a.cand_magic;
  j.cand_abs = a.cand_abs;
  j.csr = a.csr;
  j.stash = a.stash;
  j.stash_cap = a.stash_cap;
  j.stash_top = a.stash_top;
  j.tile_total = a.tile_total;
  j.tile_seg = a.tile_seg;
  j.overflow_flag = a.overflow_flag;
  const int smem = jit_wide_smem(a.r, words);
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, (const void*)kernel, 256, smem) != cudaSuccess ||
      per_sm < 1) {
    cudaGetLastError();
    return (int)cudaErrorInvalidConfiguration;
  }
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  uint64_t grid = (uint64_t)sms * per_sm;
  const uint64_t need = (a.n_tiles + 7) / 8;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  void* args[] = {&j};
  return (int)cudaLaunchKernel((const void*)kernel, dim3((unsigned)grid), dim3(256), args, (size_t)smem,
                               (cudaStream_t)stream);
}


// ---- batched decode: specialised kernel of a generated space (nullptr: generic kernel)
std::string jit_decode_source(const DecodeArgs& a) { return gen_decode_source(a); }

void* jit_decode_kernel(const DecodeArgs& a) {
  const std::string src = gen_decode_source(a);
  cudaKernel_t k = compile(src, "atf_decode_jit");
  return (void*)k;
}

int jit_decode_launch(void* kernel, const DecodeArgs& a, const uint64_t* idx, const uint64_t* digits, int64_t n,
                      int32_t* out, int64_t ld, unsigned int* bad, void* stream) {
  DecodeJitArgs j;
  std::memset(&j, 0, sizeof j);
  j.idx = idx;
  j.digits = digits;
  j.n = n;
  j.out = out;
  j.ld = ld;
  j.bad = bad;
  for (int g = 0; g < a.n_groups; g++) j.leaves[g] = a.leaves[g];
  for (int l = 0; l < a.lvl_begin[a.n_groups]; l++) j.range[l] = a.lvl_range[l];
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  int64_t blocks = (n + 255) / 256;
  if (blocks > (int64_t)sms * 8) blocks = (int64_t)sms * 8;
  if (blocks < 1) blocks = 1;
  void* args[] = {&j};
  return (int)cudaLaunchKernel((const void*)kernel, dim3((unsigned)blocks), dim3(256), args, 0, (cudaStream_t)stream);
}

}  // namespace atf

namespace atf {
void jit_set_tail_stage(int bytes) { g_tail_stage.store(bytes > 0 ? bytes : 0); }
void jit_set_tail_product(bool on) { g_tail_product.store(on); }
void jit_set_tail_leaf_direct(int mode) { g_tail_leaf_direct.store(mode); }
void jit_set_wide_group(int n) { g_wide_group.store(n); }
}  // namespace atf
