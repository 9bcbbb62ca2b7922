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
// Accept mask of one node of a tail level as a device function of the node's record words
// w[0..W): the same straight-line code as the level kernel above (field positions, constants,
// candidate magics as immediates), candidates r <= 32.  `tab` names the level's ancestor
// table arrays in the kernel parameters.  "" if the level is not covered.
std::string gen_mask_fn(const LevelArgs& a, int W, const std::vector<int32_t>& cx, const std::vector<uint32_t>& cm,
                        const std::string& fname, const std::string& tab) {
  if (a.n_terms == 0 || a.r > 32 || a.r < 1 || (int)cx.size() != a.r) return "";
  const int r = a.r;
  std::string s = "__device__ __forceinline__ u32 " + fname + "(const TailJitArgs& a, const u32* w) {\n";
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
    s += "  const u32 p" + ps + " = " + pos + ";\n";
    s += "  const i64 v" + ps + " = (i64)__ldg(a." + tab + "_range[" + ps + "] + p" + ps + ");\n";
    if (need_m[p]) s += "  const u32 g" + ps + " = __ldg(a." + tab + "_magic[" + ps + "] + p" + ps + ");\n";
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
  s += "  u32 m = " + hex(r >= 32 ? 0xffffffffu : ((1u << r) - 1u)) + ";\n";
  auto divx_bits = [&](const std::string& n) {
    std::string b = "    u32 mm = 0u;\n";
    for (int c = 0; c < r; c++)
      if (cx[c] != 0) b += "    mm |= (u32)(" + n + " * " + hex(cm[c]) + " < 0x10000u) << " + std::to_string(c) + ";\n";
    return b + "    m &= mm;\n";
  };
  for (int t = 0; t < a.n_terms; t++) {
    const Term& T = a.terms[t];
    const NfOp& oa = a.nf_op[t][0];
    const NfOp& ob = a.nf_op[t][1];
    const std::string ts = std::to_string(t);
    s += "  if (m) {  // term " + ts + "\n";
    switch (T.kind) {
      case T_DIVX:
        s += "    const u32 n" + ts + " = uabs(" + sval(oa) + ");\n" + divx_bits("n" + ts);
        break;
      case T_DIVPROD:
        s += "    const u32 av = uabs(" + sval(oa) + "), bv = uabs(" + sval(ob) + ");\n";
        s += "    const u32 ma = " + magic(oa, "av") + ";\n";
        s += "    const u32 n" + ts + " = av == 1u ? bv : __umulhi(bv, ma);\n";
        s += "    if (av == 0u || n" + ts + " * av != bv) m = 0u;\n";
        s += "    else {\n" + divx_bits("n" + ts) + "    }\n";
        break;
      case T_MULX: {
        s += "    const u32 d = uabs(" + sval(oa) + ");\n";
        s += "    const u32 md = " + magic(oa, "d") + ", md1 = md - 1u;\n";
        s += "    if (d == 0u) m = 0u;\n    else {\n      u32 mm = 0u;\n";
        for (int c = 0; c < r; c++) {
          const uint32_t ax = cx[c] < 0 ? 0u - (uint32_t)cx[c] : (uint32_t)cx[c];
          s += "      mm |= (u32)(" + hex(ax) + " * md <= md1) << " + std::to_string(c) + ";\n";
        }
        s += "      m &= mm;\n    }\n";
        break;
      }
      case T_QDIV: {
        s += "    const u32 num = uabs(" + sval(oa) + "), nb = uabs(" + sval(ob) + ");\n";
        s += "    u32 mm = 0u;\n";
        for (int c = 0; c < r; c++) {
          const uint32_t ax = cx[c] < 0 ? 0u - (uint32_t)cx[c] : (uint32_t)cx[c];
          if (ax == 0) continue;  // x == 0 rejects
          const std::string q = ax == 1 ? std::string("num") : "__umulhi(num, " + hex(cm[c]) + ")";
          s += "    if ((m >> " + std::to_string(c) + ") & 1u) { const u32 q = " + q +
               "; if (q != 0u && divisible16(nb, q)) mm |= 1u << " + std::to_string(c) + "; }\n";
        }
        s += "    m &= mm;\n";
        break;
      }
      case T_CMP: {
        static const char* rel[] = {"==", "!=", "<", "<=", ">", ">="};
        if (T.rel < R_EQ || T.rel > R_GE) return "";
        s += "    const i32 A = (i32)" + sval(oa) + ", B = (i32)" + sval(ob) + ";\n    u32 mm = 0u;\n";
        for (int c = 0; c < r; c++)
          s += "    mm |= (u32)(A * " + std::to_string(cx[c]) + " " + rel[T.rel - R_EQ] + " B) << " + std::to_string(c) + ";\n";
        s += "    m &= mm;\n";
        break;
      }
      default: return "";
    }
    s += "  }\n";
  }
  return s + "  return m;\n}\n";
}

// Kernel parameters of the generated tail kernels (same layout on both sides).
struct TailJitArgs {
  const uint32_t* parent_rec;
  uint64_t n_parents, n_tiles;
  uint32_t* tile_total;
  const uint64_t* tile_base;
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
                     u64* csr[4]; u32* rec[4];
                     const i32* l0_range[24]; const u32* l0_magic[24]; const i32* l1_range[24]; const u32* l1_magic[24];
                     const i32* l2_range[24]; const u32* l2_magic[24]; const i32* l3_range[24]; const u32* l3_magic[24]; };
)";

// Source of the two tail kernels (atf_tail_count, atf_tail_emit) for levels lv[0..nl): the
// structure of tail_count / tail_emit in expand.cuh (warp tile = 32 frontier nodes; every
// tail level processed in chunks of 32 nodes in canonical order; children staged in per-warp
// shared-memory buffers), every level's mask and child-record code specialised.  The count
// kernel runs the same chunk walk without the global writes, so no lane diverges.
std::string gen_tail_source(const TailArgs& t, int W, const std::vector<std::vector<int32_t>>& cx,
                            const std::vector<std::vector<uint32_t>>& cm) {
  const int nl = t.nl;
  if (nl < 2 || nl > kMaxTail) return "";
  std::string s = kPrelude;
  s += kTailPrelude;
  const std::string Ws = std::to_string(W);
  for (int d = 0; d < nl; d++) {
    const std::string f = gen_mask_fn(t.lv[d], W, cx[d], cm[d], "tmask" + std::to_string(d), "l" + std::to_string(d));
    if (f.empty()) return "";
    s += f;
  }
  // per-warp buffer offsets (bytes): level d holds <= 32 * r_d child records
  std::vector<int> off(nl + 1, 0);
  for (int d = 0; d < nl; d++) off[d + 1] = off[d] + ((32 * t.lv[d].r * W * 4 + 15) & ~15);
  const std::string WB = std::to_string(off[nl]);
  // chunk walk, one function per (mode, depth), deepest first
  for (int emit = 0; emit < 2; emit++) {
    for (int d = nl - 1; d >= 0; d--) {
      const std::string ds = std::to_string(d), nm = std::string(emit ? "e" : "c") + ds;
      s += "__device__ __forceinline__ void chunk_" + nm + "(const TailJitArgs& a, const u32* rec, bool valid, u64 gidx, "
           "u64* cur, unsigned char* wbuf, int lane) {\n";
      s += "  u32 m = valid ? tmask" + ds + "(a, rec) : 0u;\n";
      s += "  const u32 c = __popc(m);\n  u32 incl = c;\n";
      s += "#pragma unroll\n  for (int o = 1; o < 32; o <<= 1) { const u32 y = __shfl_up_sync(0xffffffffu, incl, o); "
           "if (lane >= o) incl += y; }\n";
      s += "  const u32 T = __shfl_sync(0xffffffffu, incl, 31);\n  u32 k = incl - c;\n  const u64 first = cur[" + ds + "];\n";
      if (emit) s += "  if (valid) a.csr[" + ds + "][gidx] = first + k;\n";
      const bool stage = emit || d + 1 < nl;
      const int fw = t.lv[d].field_word, fs = t.lv[d].field_shift;
      if (stage) {
        s += "  u32* buf = reinterpret_cast<u32*>(wbuf + " + std::to_string(off[d]) + ");\n";
        s += "  while (m) {\n    const u32 cc = __ffs(m) - 1;\n    m &= m - 1;\n";
        for (int w = 0; w < W; w++)
          s += "    buf[k * " + Ws + " + " + std::to_string(w) + "] = rec[" + std::to_string(w) + "]" +
               (w == fw ? " | (cc << " + std::to_string(fs) + ")" : "") + ";\n";
        s += "    k++;\n  }\n  __syncwarp();\n";
      }
      if (emit) {
        if (W == 1) s += "  { u32* dst = a.rec[" + ds + "] + first; for (u32 v = lane; v < T; v += 32) dst[v] = buf[v]; }\n";
        else if (W == 2)
          s += "  { uint2* dst = reinterpret_cast<uint2*>(a.rec[" + ds + "] + first * 2); const uint2* src = "
               "reinterpret_cast<const uint2*>(buf); for (u32 v = lane; v < T; v += 32) dst[v] = src[v]; }\n";
        else
          s += "  { uint4* dst = reinterpret_cast<uint4*>(a.rec[" + ds + "] + first * " + Ws + "); const uint4* src = "
               "reinterpret_cast<const uint4*>(buf); for (u32 v = lane; v < T * " + std::to_string(W / 4) +
               "; v += 32) dst[v] = src[v]; }\n";
      }
      s += "  cur[" + ds + "] = first + T;\n";
      if (d + 1 < nl) {
        s += "  for (u32 s0 = 0; s0 < T; s0 += 32) {\n    const bool v = s0 + lane < T;\n    u32 cr[" + Ws + "];\n";
        for (int w = 0; w < W; w++)
          s += "    cr[" + std::to_string(w) + "] = v ? buf[(s0 + lane) * " + Ws + " + " + std::to_string(w) + "] : 0u;\n";
        s += "    chunk_" + std::string(emit ? "e" : "c") + std::to_string(d + 1) + "(a, cr, v, first + s0 + lane, cur, wbuf, lane);\n  }\n";
      }
      if (stage) s += "  __syncwarp();\n";
      s += "}\n";
    }
  }
  // kernels
  for (int emit = 0; emit < 2; emit++) {
    const std::string kn = emit ? "atf_tail_emit" : "atf_tail_count";
    s += "extern \"C\" __global__ void __launch_bounds__(128) " + kn + "(const __grid_constant__ TailJitArgs a) {\n";
    s += "  extern __shared__ __align__(16) unsigned char smem[];\n";
    s += "  const int lane = threadIdx.x & 31;\n  unsigned char* wbuf = smem + (threadIdx.x >> 5) * " + WB + ";\n";
    s += "  const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;\n  const u64 gw = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;\n";
    if (emit) {
      s += "  if (gw == 0 && lane < " + std::to_string(nl) + ") {\n";
      s += "    const u64 above = lane == 0 ? a.n_parents : a.tile_base[(u64)(lane - 1) * (a.n_tiles + 1) + a.n_tiles];\n";
      s += "    a.csr[lane][above] = a.tile_base[(u64)lane * (a.n_tiles + 1) + a.n_tiles];\n  }\n";
    }
    s += "  for (u64 tile = gw; tile < a.n_tiles; tile += nw) {\n    u64 cur[" + std::to_string(nl) + "];\n";
    for (int d = 0; d < nl; d++)
      s += emit ? "    cur[" + std::to_string(d) + "] = a.tile_base[(u64)" + std::to_string(d) + " * (a.n_tiles + 1) + tile];\n"
                : "    cur[" + std::to_string(d) + "] = 0;\n";
    s += "    const u64 nd = tile * 32 + lane;\n    const bool v = nd < a.n_parents;\n    u32 rec[" + Ws + "];\n";
    s += "    for (int w = 0; w < " + Ws + "; w++) rec[w] = v ? __ldg(a.parent_rec + nd * " + Ws + " + w) : 0u;\n";
    s += std::string("    chunk_") + (emit ? "e" : "c") + "0(a, rec, v, nd, cur, wbuf, lane);\n";
    if (!emit)
      for (int d = 0; d < nl; d++)
        s += "    if (lane == 0) a.tile_total[(u64)" + std::to_string(d) + " * a.n_tiles + tile] = (u32)cur[" +
             std::to_string(d) + "];\n";
    s += "  }\n}\n";
  }
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
  int warp_bytes = 0, per_sm = 0;
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
                            const std::vector<std::vector<uint32_t>>& cand_magics) {
  return gen_tail_source(t, words, cand_values, cand_magics);
}

void* jit_tail_kernels(const TailArgs& t, int words, const std::vector<std::vector<int32_t>>& cand_values,
                       const std::vector<std::vector<uint32_t>>& cand_magics) {
  const std::string src = gen_tail_source(t, words, cand_values, cand_magics);
  if (src.empty()) return nullptr;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_tails.find(src);
    if (it != g_tails.end()) return it->second.count ? (void*)&it->second : nullptr;
  }
  TailJit tj;
  tj.count = compile(src, "atf_tail_count");
  tj.emit = compile(src, "atf_tail_emit");
  int wb = 0;
  for (int d = 0; d < t.nl; d++) wb += (32 * t.lv[d].r * words * 4 + 15) & ~15;
  tj.warp_bytes = wb;
  if (tj.count && tj.emit) {
    const int smem = 4 * wb;
    bool ok = true;
    for (cudaKernel_t k : {tj.count, tj.emit}) {
      if (smem > 48 * 1024 &&
          cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
        ok = false;
    }
    int per_sm = 0;
    if (ok && cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, (const void*)tj.emit, 128, smem) != cudaSuccess)
      ok = false;
    cudaGetLastError();
    tj.per_sm = per_sm;
    if (!ok || per_sm < 1) tj.count = tj.emit = nullptr;
  } else {
    tj.count = tj.emit = nullptr;
  }
  std::lock_guard<std::mutex> lk(g_mu);
  TailJit& slot = g_tails[src];
  slot = tj;
  return slot.count ? (void*)&slot : nullptr;
}

int jit_tail_launch(void* handle, const TailArgs& t, bool emit, void* stream) {
  const TailJit& tj = *reinterpret_cast<const TailJit*>(handle);
  TailJitArgs j;
  std::memset(&j, 0, sizeof j);
  j.parent_rec = t.parent_rec;
  j.n_parents = t.n_parents;
  j.n_tiles = t.n_tiles;
  j.tile_total = t.tile_total;
  j.tile_base = t.tile_base;
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
  uint64_t grid = (uint64_t)sms * tj.per_sm;
  const uint64_t need = (t.n_tiles + 3) / 4;  // 4 warps per CTA, one warp tile each
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  void* args[] = {&j};
  cudaError_t e = cudaLaunchKernel((const void*)(emit ? tj.emit : tj.count), dim3((unsigned)grid), dim3(128), args,
                                   (size_t)(4 * tj.warp_bytes), (cudaStream_t)stream);
  return (int)e;
}

}  // namespace atf
