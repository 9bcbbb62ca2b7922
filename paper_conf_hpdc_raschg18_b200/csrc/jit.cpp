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

std::mutex g_mu;
std::unordered_map<std::string, cudaKernel_t> g_cache;  // source -> kernel (nullptr: failed)

cudaKernel_t compile(const std::string& src) {
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_cache.find(src);
    if (it != g_cache.end()) return it->second;
  }
  Nvrtc& nv = nvrtc();
  cudaKernel_t k = nullptr;
  if (nv.ok) {
    nvrtcProgram_ prog = nullptr;
    if (nv.create(&prog, src.c_str(), "atf_level.cu", 0, nullptr, nullptr) == 0) {
      const char* opts[] = {"-arch=sm_100a", "-std=c++17", "-default-device", "-lineinfo"};
      if (nv.compile(prog, 4, opts) == 0) {
        size_t n = 0;
        nv.cubin_size(prog, &n);
        std::vector<char> cubin(n);
        nv.cubin(prog, cubin.data());
        cudaLibrary_t lib = nullptr;
        if (cudaLibraryLoadData(&lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0) == cudaSuccess) {
          if (cudaLibraryGetKernel(&k, lib, "atf_nfast_jit") != cudaSuccess) k = nullptr;
        }
        cudaGetLastError();
      } else if (getenv("ATF_JIT_VERBOSE") && nv.log_size && nv.log) {
        size_t n = 0;
        nv.log_size(prog, &n);
        std::string log(n, '\0');
        nv.log(prog, &log[0]);
        fprintf(stderr, "atfgen jit: compile failed:\n%s\n%s\n", log.c_str(), src.c_str());
      }
      nv.destroy(&prog);
    }
  }
  std::lock_guard<std::mutex> lk(g_mu);
  g_cache[src] = k;
  return k;
}

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
  if (getenv("ATF_NO_JIT")) return nullptr;
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

}  // namespace atf
