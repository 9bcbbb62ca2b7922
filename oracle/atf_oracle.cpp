// ============================================================================
// atf_oracle — the CPU ORACLE for ATF search-space generation.
//
// TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
// bench.py's cpu_baseline / --impl reference legs may build, call or execute
// anything under oracle/.  The product path (paper_conf_hpdc_raschg18_b200/)
// never does, and this file shares no code with it: it parses the spec JSON
// itself and has its own bytecode interpreter.
//
// What it computes (PAPER.md = P:n):
//   * The search space is the set of tuples (v_1..v_P) in R_1 x ... x R_P for
//     which every parameter's constraint holds ("The generated search
//     space comprises all valid parameter configurations, i.e., for which the
//     parameters' constraints are satisfied").
//   * O1 = CLTune-style generation: iterate the entire unconstrained product and
//     filter ("CLTune iterates over the entire, unconstrained search
//     space and then filters out the invalid configurations").
//   * O2 = ATF-style generation: iterate each parameter's constrained range given
//     the earlier parameters ("ATF filters out invalid
//     configurations by iterating over the constrained ranges"), per group of
//     interdependent parameters.  O2 records f_k (accepted level-k
//     prefixes, dead ends included) and evals_k = f_{k-1} * r_k.
//   * S = product of group sizes, as unsigned __int128.
//   * decode(i): OpenTuner's TP indexes "the configuration with index TP within
//     the ATF search space".  Convention (readings #4,#11):
//     0-based, mixed radix over groups with group 0 (earliest first member) most
//     significant, lexicographic range-position order inside a group.
//
// Readings of unclear points follow SURVEY.md §8(c) (listed in DESIGN.md):
//   intervals inclusive (#1), value = gen(begin + k*step) (#2), pow2 = exact
//   2^i (#3), sets in listed order, duplicates rejected (#5), alias semantics
//   (#6), strict evaluation with any zero divisor => candidate rejected (#7),
//   C truncating division (#8), exact int64 arithmetic, overflow = error (#9),
//   backward references only (#10).
//
// Parity status of each function is stated in DESIGN.md ("Oracle pins").
// ============================================================================
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cinttypes>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <functional>
#include <map>
#include <sstream>
#include <stdexcept>
#include <string>
#include <numeric>
#include <thread>
#include <vector>

using i64 = int64_t;
using u64 = uint64_t;
using u128 = unsigned __int128;

// ---------------------------------------------------------------- tiny JSON
struct Json {
  enum Kind { NUL, NUM, STR, ARR, OBJ, BOOL } kind = NUL;
  i64 num = 0;
  bool integral = true;  // NUM without fraction / exponent
  bool b = false;
  std::string str;
  std::vector<Json> arr;
  std::vector<std::pair<std::string, Json>> obj;
  const Json& at(const std::string& k) const {
    for (auto& kv : obj)
      if (kv.first == k) return kv.second;
    throw std::runtime_error("json: missing key " + k);
  }
  bool has(const std::string& k) const {
    for (auto& kv : obj)
      if (kv.first == k) return true;
    return false;
  }
};

struct JsonParser {
  const std::string& s;
  size_t i = 0;
  explicit JsonParser(const std::string& src) : s(src) {}
  void ws() { while (i < s.size() && isspace((unsigned char)s[i])) i++; }
  Json parse() {
    ws();
    if (i >= s.size()) throw std::runtime_error("json: eof");
    char c = s[i];
    Json j;
    if (c == '{') {
      j.kind = Json::OBJ; i++; ws();
      if (s[i] == '}') { i++; return j; }
      for (;;) {
        ws(); Json k = parse(); ws();
        if (s[i] != ':') throw std::runtime_error("json: expected :");
        i++;
        Json v = parse();
        j.obj.emplace_back(k.str, v);
        ws();
        if (s[i] == ',') { i++; continue; }
        if (s[i] == '}') { i++; break; }
        throw std::runtime_error("json: expected , or }");
      }
    } else if (c == '[') {
      j.kind = Json::ARR; i++; ws();
      if (s[i] == ']') { i++; return j; }
      for (;;) {
        j.arr.push_back(parse()); ws();
        if (s[i] == ',') { i++; continue; }
        if (s[i] == ']') { i++; break; }
        throw std::runtime_error("json: expected , or ]");
      }
    } else if (c == '"') {
      j.kind = Json::STR; i++;
      while (s[i] != '"') {
        if (s[i] == '\\') i++;
        j.str.push_back(s[i++]);
      }
      i++;
    } else if (c == 't' || c == 'f') {
      j.kind = Json::BOOL; j.b = (c == 't'); i += j.b ? 4 : 5;
    } else if (c == 'n') {
      i += 4;
    } else {
      j.kind = Json::NUM;
      size_t st = i;
      if (s[i] == '-') i++;
      while (i < s.size() && isdigit((unsigned char)s[i])) i++;
      j.num = std::stoll(s.substr(st, i - st));
      // a fraction / exponent (display metadata such as the float values of atfspec.floats):
      // consumed and marked; a spec field read as an integer rejects it
      if (i < s.size() && (s[i] == '.' || s[i] == 'e' || s[i] == 'E')) {
        j.integral = false;
        while (i < s.size() && (isdigit((unsigned char)s[i]) || s[i] == '.' || s[i] == 'e' || s[i] == 'E' ||
                                s[i] == '+' || s[i] == '-'))
          i++;
      }
    }
    return j;
  }
};

// ---------------------------------------------------------------- the spec
enum Op {
  X = 1, PARAM = 2, CONST = 3, ADD = 4, SUB = 5, MUL = 6, DIV = 7, MOD = 8, MIN = 9, MAX = 10,
  EQ = 11, NE = 12, LT = 13, LE = 14, GT = 15, GE = 16, DIVIDES = 17, MULOF = 18,
  AND = 19, OR = 20, NOT = 21
};

struct Param {
  std::string name;
  std::vector<i64> values;                    // materialised range, in range order
  std::vector<std::vector<int32_t>> programs; // ANDed constraint programs
  std::vector<int> refs;                      // params referenced by the programs
};

struct Spec {
  std::string name;
  std::vector<Param> params;
};

static i64 run_value(const std::vector<int32_t>& code, i64 x, const i64* vals, bool& poison);

// "atf::interval<T>(begin, end, step_size, generator) represents the values
// ... from begin to end using the optional step_size"; "the interval comprises the
// elements generator(i) for each i from begin to end"; "atf::set(val_1,...,val_n)".
static std::vector<i64> materialise(const Json& r) {
  // values are int64 ("arbitrary fundamental type T"; reading #22): an index
  // or value outside int64 is an error
  std::string kind = r.at("kind").str;
  std::vector<i64> v;
  if (kind == "interval" || kind == "pow2") {
    i64 b = r.at("begin").num, e = r.at("end").num, st = r.at("step").num;
    if (st <= 0) throw std::runtime_error("range: step must be positive");
    for (__int128 i = b; i <= e; i += st) {     // inclusive both ends (reading #1)
      if (kind == "interval") {
        v.push_back((i64)i);
      } else {
        if (i < 0 || i > 62) throw std::runtime_error("range: pow2 exponent outside [0,62]");
        i64 p = 1;
        for (i64 k = 0; k < (i64)i; k++) p *= 2;  // exact 2^i (reading #3)
        v.push_back(p);
      }
    }
  } else if (kind == "gen") {                   // P:57 generator(i), i = begin, begin+step, ..., <= end
    i64 b = r.at("begin").num, e = r.at("end").num, st = r.at("step").num;
    if (st <= 0) throw std::runtime_error("range: step must be positive");
    std::vector<int32_t> code;
    for (auto& w : r.at("code").arr) code.push_back((int32_t)w.num);
    for (size_t k = 0; k < code.size(); k += (code[k] == CONST ? 3 : 1))
      if (code[k] == PARAM) throw std::runtime_error("range: generator references a parameter");
    for (__int128 i = b; i <= e; i += st) {
      bool poison = false;
      i64 y = run_value(code, (i64)i, nullptr, poison);
      if (poison) throw std::runtime_error("range: generator poison");
      for (i64 z : v)
        if (z == y) throw std::runtime_error("range: duplicate generator value");  // reading #5
      v.push_back(y);
    }
  } else if (kind == "set") {
    for (auto& x : r.at("values").arr) {
      if (x.kind != Json::NUM || !x.integral) throw std::runtime_error("range: set values must be integers");
      for (i64 y : v)
        if (y == x.num) throw std::runtime_error("range: duplicate set value");  // reading #5
      v.push_back(x.num);
    }
  } else {
    throw std::runtime_error("range: unknown kind " + kind);
  }
  return v;
}

// Value width of the files this oracle reads and writes (o1 / leaves / decode rows, check
// input): int32 while every value of the spec fits int32, else int64 (reading #22).
static bool g_w64 = false;
static void put_val(FILE* f, i64 v) {
  if (g_w64) {
    std::fwrite(&v, 8, 1, f);
  } else {
    int32_t w = (int32_t)v;
    std::fwrite(&w, 4, 1, f);
  }
}

static Spec load_spec(const std::string& path) {
  std::ifstream f(path);
  if (!f) throw std::runtime_error("cannot open " + path);
  std::stringstream ss;
  ss << f.rdbuf();
  std::string txt = ss.str();
  JsonParser jp(txt);
  Json j = jp.parse();
  Spec s;
  s.name = j.at("name").str;
  for (auto& pj : j.at("params").arr) {
    Param p;
    p.name = pj.at("name").str;
    for (auto& q : s.params)
      if (q.name == p.name) throw std::runtime_error("duplicate parameter name " + p.name);  // P:53 unique
    p.values = materialise(pj.at("range"));
    if (pj.has("constraints"))
      for (auto& cj : pj.at("constraints").arr) {
        std::vector<int32_t> code;
        for (auto& w : cj.arr) code.push_back((int32_t)w.num);
        p.programs.push_back(code);
      }
    int self = (int)s.params.size();
    for (auto& code : p.programs)
      for (size_t i = 0; i < code.size();) {
        int op = code[i];
        if (op == PARAM) {
          int jd = code[i + 1];
          if (jd < 0 || jd >= self) throw std::runtime_error("constraint references a later parameter");  // reading #10
          if (std::find(p.refs.begin(), p.refs.end(), jd) == p.refs.end()) p.refs.push_back(jd);
          i += 2;
        } else if (op == CONST) {
          i += 3;
        } else {
          i += 1;
        }
      }
    for (i64 v : p.values)
      if (v < INT32_MIN || v > INT32_MAX) g_w64 = true;
    s.params.push_back(p);
  }
  return s;
}

// ---------------------------------------------------------------- interpreter
// postfix int32 words, int64 stack.  The candidate is accepted
// iff no poison occurred and exactly one nonzero item remains.  Poison: a zero
// divisor anywhere (DIV/MOD by 0, DIVIDES with a=0, MULOF with b=0) — reading #7.
// Evaluation is strict: every operation of the program is executed.
static std::atomic<bool> g_overflow{false};

static i64 run_value(const std::vector<int32_t>& code, i64 x, const i64* vals, bool& poison) {
  i64 st[256];
  int sp = 0;
  for (size_t i = 0; i < code.size();) {
    int op = code[i];
    if (op == X) { st[sp++] = x; i++; continue; }
    if (op == PARAM) { st[sp++] = vals[code[i + 1]]; i += 2; continue; }
    if (op == CONST) {
      u64 lo = (uint32_t)code[i + 1], hi = (uint32_t)code[i + 2];
      st[sp++] = (i64)((hi << 32) | lo);
      i += 3;
      continue;
    }
    if (op == NOT) { st[sp - 1] = (st[sp - 1] == 0); i++; continue; }
    if (sp < 2) throw std::runtime_error("bytecode: stack underflow");
    i64 b = st[--sp];
    i64 a = st[--sp];
    i64 r = 0;
    switch (op) {
      case ADD: if (__builtin_add_overflow(a, b, &r)) g_overflow = true; break;
      case SUB: if (__builtin_sub_overflow(a, b, &r)) g_overflow = true; break;
      case MUL: if (__builtin_mul_overflow(a, b, &r)) g_overflow = true; break;
      case DIV:
        if (b == 0) { poison = true; r = 0; }
        else if (a == INT64_MIN && b == -1) { g_overflow = true; r = 0; }
        else r = a / b;                              // C truncation (reading #8)
        break;
      case MOD:
        if (b == 0) { poison = true; r = 0; }
        else if (b == -1) r = 0;
        else r = a % b;
        break;
      case MIN: r = a < b ? a : b; break;
      case MAX: r = a > b ? a : b; break;
      case EQ: r = (a == b); break;
      case NE: r = (a != b); break;
      case LT: r = (a < b); break;
      case LE: r = (a <= b); break;
      case GT: r = (a > b); break;
      case GE: r = (a >= b); break;
      case DIVIDES:                                  // a b -> [a != 0 and b mod a == 0]
        if (a == 0) { poison = true; r = 0; }
        else r = (a == -1) ? 1 : (b % a == 0);
        break;
      case MULOF:                                    // a b -> [b != 0 and a mod b == 0]
        if (b == 0) { poison = true; r = 0; }
        else r = (b == -1) ? 1 : (a % b == 0);
        break;
      case AND: r = (a != 0) && (b != 0); break;     // strict: both operands already evaluated
      case OR: r = (a != 0) || (b != 0); break;
      default: throw std::runtime_error("bytecode: bad opcode " + std::to_string(op));
    }
    st[sp++] = r;
    i++;
  }
  if (sp != 1) throw std::runtime_error("bytecode: program must leave exactly one item");
  return st[0];
}

static bool run_program(const std::vector<int32_t>& code, i64 x, const i64* vals) {
  bool poison = false;
  const i64 v = run_value(code, x, vals, poison);
  return !poison && v != 0;
}

// Optional hand-written predicates (native C++ encodings of C1, C2, C3, saxpy) used
// to pin the bytecode encodings: both must agree on every evaluated candidate.
using NativePred = std::function<bool(int, i64, const i64*)>;
static NativePred g_native;
static bool g_native_check = false;
static std::atomic<u64> g_native_mismatch{0};

static NativePred make_native(const std::string& spec) {
  // spec = "c1" | "c2:N" | "c3:M,N,K" | "saxpy:N"
  auto nums = [&](size_t from) {
    std::vector<i64> v;
    std::stringstream ss(spec.substr(from));
    std::string t;
    while (std::getline(ss, t, ',')) v.push_back(std::stoll(t));
    return v;
  };
  auto dv = [](i64 a, i64 b) { return a != 0 && b % a == 0; };  // "a divides b"
  if (spec == "c1") {
    return [dv](int p, i64 x, const i64* v) {
      if (p == 0) return dv(x, 64);
      return dv(x, 64) && v[0] * x <= 1024;
    };
  }
  if (spec.rfind("c2:", 0) == 0) {
    i64 N = nums(3)[0];
    return [dv, N](int p, i64 x, const i64* v) {
      const i64 WGD = v[0], MDIMCD = v[1], NDIMCD = v[2], MDIMAD = v[3], NDIMBD = v[4];
      switch (p) {
        case 0: return dv(x, N) && dv(x, N);
        case 1: case 2: case 5: return dv(x, WGD);
        case 3: case 4: { i64 q = x ? MDIMCD * NDIMCD / x : 0; return x != 0 && q != 0 && dv(x, WGD) && WGD % q == 0; }
        case 6: return dv(MDIMCD * x, WGD) && dv(MDIMAD * x, WGD);
        case 7: return dv(NDIMCD * x, WGD) && dv(NDIMBD * x, WGD);
        default: return true;
      }
    };
  }
  if (spec.rfind("c3:", 0) == 0) {
    return [dv](int p, i64 x, const i64* v) {
      const i64 MWG = v[0], NWG = v[1], KWG = v[2], MDIMC = v[3], NDIMC = v[4], MDIMA = v[5], NDIMB = v[6];
      switch (p) {
        case 3: return dv(x, MWG);
        case 4: return dv(x, NWG);
        case 5: { i64 q = x ? MDIMC * NDIMC / x : 0; return x != 0 && q != 0 && dv(x, MWG) && KWG % q == 0; }
        case 6: { i64 q = x ? MDIMC * NDIMC / x : 0; return x != 0 && q != 0 && dv(x, NWG) && KWG % q == 0; }
        case 7: return dv(x, KWG);
        case 8: return dv(MDIMC * x, MWG) && dv(MDIMA * x, MWG);
        case 9: return dv(NDIMC * x, NWG) && dv(NDIMB * x, NWG);
        default: return true;
      }
    };
  }
  if (spec.rfind("saxpy:", 0) == 0) {
    i64 N = nums(6)[0];
    return [dv, N](int p, i64 x, const i64* v) {
      if (p == 0) return dv(x, N);
      return v[0] != 0 && dv(x, N / v[0]);
    };
  }
  throw std::runtime_error("unknown --native " + spec);
}

// constraint of parameter p (all programs ANDed) for candidate value x, given the
// values of the already-fixed parameters (indexed by parameter id).
static bool constraint_holds(const Spec& s, int p, i64 x, const i64* vals) {
  if (g_native && !g_native_check) return g_native(p, x, vals);
  bool ok = true;
  for (auto& code : s.params[p].programs) ok = run_program(code, x, vals) && ok;  // strict AND
  if (g_native_check && g_native(p, x, vals) != ok) g_native_mismatch++;
  return ok;
}

// ---------------------------------------------------------------- groups
// parameters whose constraints do not interact form independent groups.
// Groups = connected components of the undirected graph p -- q for every q that
// p's constraints reference.  Order: by first (lowest-id) member; members in
// declaration order.
static std::vector<std::vector<int>> groups_of(const Spec& s) {
  int n = (int)s.params.size();
  std::vector<std::vector<int>> adj(n);
  for (int p = 0; p < n; p++)
    for (int q : s.params[p].refs) { adj[p].push_back(q); adj[q].push_back(p); }
  std::vector<int> comp(n, -1);
  std::vector<std::vector<int>> groups;
  for (int p = 0; p < n; p++) {
    if (comp[p] >= 0) continue;
    int g = (int)groups.size();
    groups.push_back({});
    std::vector<int> stack{p};
    comp[p] = g;
    while (!stack.empty()) {
      int u = stack.back(); stack.pop_back();
      groups[g].push_back(u);
      for (int v : adj[u]) if (comp[v] < 0) { comp[v] = g; stack.push_back(v); }
    }
    std::sort(groups[g].begin(), groups[g].end());
  }
  return groups;
}

// ---------------------------------------------------------------- O2 per group
struct LevelStats { u64 evals = 0, f = 0; };

struct GroupRun {
  const Spec* s;
  std::vector<int> members;
  std::vector<LevelStats> lv;
  // leaf sink: called with the values of the group's members (group order)
  std::function<void(const i64* gvals)> sink;
  std::vector<i64> vals;   // by parameter id
  std::vector<i64> gvals;  // by group level

  void rec(size_t k) {
    int p = members[k];
    const auto& R = s->params[p].values;
    for (size_t j = 0; j < R.size(); j++) {
      lv[k].evals++;
      i64 x = R[j];
      if (!constraint_holds(*s, p, x, vals.data())) continue;
      lv[k].f++;
      vals[p] = x;
      gvals[k] = x;
      if (k + 1 == members.size()) { if (sink) sink(gvals.data()); }
      else rec(k + 1);
    }
  }
  // run O2 restricted to level-1 positions [j0, j1)
  void run(size_t j0, size_t j1) {
    lv.assign(members.size(), LevelStats{});
    vals.assign(s->params.size(), 0);
    gvals.assign(members.size(), 0);
    int p = members[0];
    const auto& R = s->params[p].values;
    for (size_t j = j0; j < j1 && j < R.size(); j++) {
      lv[0].evals++;
      i64 x = R[j];
      if (!constraint_holds(*s, p, x, vals.data())) continue;
      lv[0].f++;
      vals[p] = x;
      gvals[0] = x;
      if (members.size() == 1) { if (sink) sink(gvals.data()); }
      else rec(1);
    }
  }
};

// order-dependent hash of a row sequence: H = sum_i rowhash(row_i) * (2 i + 1) mod 2^64
static inline u64 rowhash(const i64* v, size_t n) {
  u64 z = 0x243F6A8885A308D3ull;
  for (size_t k = 0; k < n; k++) {
    z ^= g_w64 ? (u64)v[k] : (u64)(uint32_t)(int32_t)v[k];
    z *= 0x9E3779B97F4A7C15ull;
    z ^= z >> 32;
  }
  return z;
}

struct ChunkResult {
  std::vector<LevelStats> lv;
  u64 a = 0, b = 0, n = 0;   // hash partials: sum rh*(2 li + 1), sum rh, leaf count
};

// O2 over a whole group, level-1 positions distributed dynamically over threads;
// per-position results are combined in position order (deterministic).
static std::vector<ChunkResult> run_group_parallel(const Spec& s, const std::vector<int>& members,
                                                   int threads, bool want_hash) {
  size_t r1 = s.params[members[0]].values.size();
  std::vector<ChunkResult> res(r1);
  std::atomic<size_t> next{0};
  auto worker = [&]() {
    GroupRun gr;
    gr.s = &s;
    gr.members = members;
    for (;;) {
      size_t j = next.fetch_add(1);
      if (j >= r1) break;
      ChunkResult& cr = res[j];
      if (want_hash)
        gr.sink = [&cr, &members](const i64* gv) {
          u64 rh = rowhash(gv, members.size());
          cr.a += rh * (2 * cr.n + 1);
          cr.b += rh;
          cr.n++;
        };
      else
        gr.sink = [&cr](const i64*) { cr.n++; };
      gr.run(j, j + 1);
      cr.lv = gr.lv;
    }
  };
  std::vector<std::thread> th;
  for (int t = 0; t < std::max(1, threads); t++) th.emplace_back(worker);
  for (auto& t : th) t.join();
  return res;
}

static std::string u128_str(u128 v) {
  if (v == 0) return "0";
  std::string s;
  while (v) { s.push_back('0' + (int)(v % 10)); v /= 10; }
  std::reverse(s.begin(), s.end());
  return s;
}


// ---------------------------------------------------------------- commands
static int cmd_info(const Spec& s, int threads, bool want_hash) {
  auto groups = groups_of(s);
  u128 S = 1, U = 1;
  bool Sover = false, Uover = false;
  std::printf("{\"name\":\"%s\",\"params\":[", s.name.c_str());
  for (size_t p = 0; p < s.params.size(); p++) {
    std::printf("%s{\"name\":\"%s\",\"r\":%zu}", p ? "," : "", s.params[p].name.c_str(), s.params[p].values.size());
    u128 r = s.params[p].values.size();
    if (r && U > (~(u128)0) / r) Uover = true; else U *= r;
  }
  std::printf("],\"groups\":[");
  double gen_s = 0;  // O2 generation time (steady clock; spec parsing and printing excluded)
  for (size_t g = 0; g < groups.size(); g++) {
    const auto tg = std::chrono::steady_clock::now();
    auto res = run_group_parallel(s, groups[g], threads, want_hash);
    gen_s += std::chrono::duration<double>(std::chrono::steady_clock::now() - tg).count();
    size_t L = groups[g].size();
    std::vector<LevelStats> lv(L);
    u64 n = 0, H = 0;
    for (auto& cr : res) {
      for (size_t k = 0; k < L && k < cr.lv.size(); k++) { lv[k].evals += cr.lv[k].evals; lv[k].f += cr.lv[k].f; }
      H += cr.a + 2 * n * cr.b;   // shift chunk-local indices by the leaves before it
      n += cr.n;
    }
    // a level-1 position with no work still counts one evaluation (handled by run())
    std::printf("%s{\"members\":[", g ? "," : "");
    for (size_t k = 0; k < L; k++) std::printf("%s%d", k ? "," : "", groups[g][k]);
    std::printf("],\"levels\":[");
    for (size_t k = 0; k < L; k++)
      std::printf("%s{\"param\":%d,\"r\":%zu,\"evals\":%" PRIu64 ",\"f\":%" PRIu64 "}", k ? "," : "", groups[g][k],
                  s.params[groups[g][k]].values.size(), lv[k].evals, lv[k].f);
    std::printf("],\"size\":%" PRIu64, n);
    if (want_hash) std::printf(",\"hash\":\"%" PRIu64 "\"", H);
    std::printf("}");
    if (n && S > (~(u128)0) / n) Sover = true; else S *= n;
  }
  std::printf("],\"S\":\"%s\",\"unconstrained\":\"%s\"", Sover ? "overflow" : u128_str(S).c_str(),
              Uover ? "overflow" : u128_str(U).c_str());
  if (g_native_check) std::printf(",\"native_mismatch\":%" PRIu64, (u64)g_native_mismatch.load());
  std::printf(",\"gen_seconds\":%.6f,\"threads\":%d", gen_s, threads);
  std::printf(",\"overflow\":%s}\n", g_overflow ? "true" : "false");
  return 0;
}

// O1: the literal brute force over the full, unfiltered product (declaration order
// odometer); then rows are sorted by the canonical group-major position key.
static int cmd_o1(const Spec& s, const char* out) {
  size_t P = s.params.size();
  auto groups = groups_of(s);
  std::vector<size_t> pos(P, 0);
  std::vector<i64> vals(P);
  for (size_t p = 0; p < P; p++) if (s.params[p].values.empty()) { P = 0; }
  struct Row { std::vector<u64> key; std::vector<i64> vals; };
  std::vector<Row> rows;
  u64 evaluated = 0;
  const auto t0 = std::chrono::steady_clock::now();
  if (P == s.params.size() && P > 0) {
    for (;;) {
      for (size_t p = 0; p < P; p++) vals[p] = s.params[p].values[pos[p]];
      evaluated++;
      bool ok = true;
      for (size_t p = 0; p < P; p++) ok = constraint_holds(s, (int)p, vals[p], vals.data()) && ok;
      if (ok) {
        Row r;
        for (auto& g : groups) for (int q : g) r.key.push_back(pos[q]);
        r.vals = vals;
        rows.push_back(std::move(r));
      }
      size_t p = P;   // odometer, last parameter fastest
      while (p > 0) {
        p--;
        if (++pos[p] < s.params[p].values.size()) break;
        pos[p] = 0;
        if (p == 0) { p = SIZE_MAX; break; }
      }
      if (p == SIZE_MAX) break;
    }
  }
  std::stable_sort(rows.begin(), rows.end(), [](const Row& a, const Row& b) { return a.key < b.key; });
  const double o1_s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  if (out) {
    FILE* f = std::fopen(out, "wb");
    for (auto& r : rows)
      for (i64 v : r.vals) put_val(f, v);
    std::fclose(f);
  }
  std::printf("{\"S\":%zu,\"evaluated\":%" PRIu64 ",\"seconds\":%.6f,\"overflow\":%s}\n", rows.size(), evaluated,
              o1_s, g_overflow ? "true" : "false");
  return 0;
}

// leaves of group g in canonical order: int32 rows of the group's member values
static int cmd_leaves(const Spec& s, int g, const char* out) {
  auto groups = groups_of(s);
  GroupRun gr;
  gr.s = &s;
  gr.members = groups.at(g);
  FILE* f = std::fopen(out, "wb");
  u64 n = 0;
  gr.sink = [&](const i64* gv) {
    for (size_t k = 0; k < gr.members.size(); k++) put_val(f, gv[k]);
    n++;
  };
  gr.run(0, SIZE_MAX);
  std::fclose(f);
  std::printf("{\"group\":%d,\"size\":%" PRIu64 "}\n", g, n);
  return 0;
}

// decode: indices (u64 little-endian file) -> values, int32 SoA [P][n] (int64 if g_w64; invalid
// rows INT32_MIN / INT64_MIN).  Streams each
// group in canonical order and picks the requested digits (no materialisation).
static int cmd_decode(const Spec& s, const char* idxfile, const char* out, int threads) {
  auto groups = groups_of(s);
  size_t G = groups.size(), P = s.params.size();
  std::vector<u64> sizes(G);
  for (size_t g = 0; g < G; g++) {
    auto res = run_group_parallel(s, groups[g], threads, false);
    u64 n = 0;
    for (auto& cr : res) n += cr.n;
    sizes[g] = n;
  }
  u128 S = 1;
  for (u64 z : sizes) S *= z;
  std::vector<u64> idx;
  {
    FILE* f = std::fopen(idxfile, "rb");
    u64 v;
    while (std::fread(&v, 8, 1, f) == 1) idx.push_back(v);
    std::fclose(f);
  }
  size_t n = idx.size();
  std::vector<i64> res(P * n, g_w64 ? INT64_MIN : (i64)INT32_MIN);
  u64 bad = 0;
  // digits: group G-1 least significant
  std::vector<std::vector<u64>> digit(G, std::vector<u64>(n));
  std::vector<char> valid(n, 1);
  for (size_t i = 0; i < n; i++) {
    if ((u128)idx[i] >= S) { valid[i] = 0; bad++; continue; }
    u128 rem = idx[i];
    for (size_t g = G; g-- > 0;) { digit[g][i] = (u64)(rem % sizes[g]); rem /= sizes[g]; }
  }
  for (size_t g = 0; g < G; g++) {
    std::vector<size_t> order;
    for (size_t i = 0; i < n; i++) if (valid[i]) order.push_back(i);
    std::sort(order.begin(), order.end(), [&](size_t a, size_t b) { return digit[g][a] < digit[g][b]; });
    size_t cur = 0;
    u64 leaf = 0;
    GroupRun gr;
    gr.s = &s;
    gr.members = groups[g];
    gr.sink = [&](const i64* gv) {
      while (cur < order.size() && digit[g][order[cur]] == leaf) {
        for (size_t k = 0; k < gr.members.size(); k++) res[(size_t)gr.members[k] * n + order[cur]] = gv[k];
        cur++;
      }
      leaf++;
    };
    gr.run(0, SIZE_MAX);
  }
  // order-dependent hash of the decoded rows (row i = values of index i, all params)
  u64 H = 0;
  std::vector<i64> row(P);
  for (size_t i = 0; i < n; i++) {
    for (size_t p = 0; p < P; p++) row[p] = res[p * n + i];
    H += rowhash(row.data(), P) * (2 * (u64)i + 1);
  }
  if (std::strcmp(out, "-") != 0) {
    FILE* f = std::fopen(out, "wb");
    for (i64 v : res) put_val(f, v);
    std::fclose(f);
  }
  std::printf("{\"n\":%zu,\"invalid\":%" PRIu64 ",\"S\":\"%s\",\"hash\":\"%" PRIu64 "\"}\n", n, bad,
              u128_str(S).c_str(), H);
  return 0;
}

// check: rows of values (int32 [n][P], int64 if g_w64) -> how many satisfy every constraint
static int cmd_check(const Spec& s, const char* rowfile, const char* flagfile) {
  size_t P = s.params.size();
  FILE* f = std::fopen(rowfile, "rb");
  FILE* ff = flagfile ? std::fopen(flagfile, "wb") : nullptr;  // optional: one byte per row
  std::vector<int32_t> row(P);
  std::vector<i64> row64(P);
  std::vector<i64> vals(P);
  u64 n = 0, ok = 0, in_range = 0;
  for (;;) {
    if (g_w64 ? std::fread(row64.data(), 8, P, f) != P : std::fread(row.data(), 4, P, f) != P) break;
    n++;
    bool good = true, inr = true;
    for (size_t p = 0; p < P; p++) {
      vals[p] = g_w64 ? row64[p] : (i64)row[p];
      auto& R = s.params[p].values;
      if (std::find(R.begin(), R.end(), vals[p]) == R.end()) inr = false;
    }
    for (size_t p = 0; p < P; p++) good = constraint_holds(s, (int)p, vals[p], vals.data()) && good;
    ok += (good && inr);
    in_range += inr;
    if (ff) std::fputc((good && inr) ? 1 : 0, ff);
  }
  std::fclose(f);
  if (ff) std::fclose(ff);
  std::printf("{\"rows\":%" PRIu64 ",\"valid\":%" PRIu64 ",\"in_range\":%" PRIu64 "}\n", n, ok, in_range);
  return 0;
}

// time: O2 on a bounded sample — groups in order, level-1 positions in order, until
// the CPU budget is spent.  Reports evals and leaves generated and the wall time.
static int cmd_time(const Spec& s, int threads, double budget_s) {
  auto groups = groups_of(s);
  u64 evals = 0, leaves = 0, l1_done = 0, l1_total = 0;
  auto t0 = std::chrono::steady_clock::now();
  bool stop = false;
  for (auto& members : groups) {
    size_t r1 = s.params[members[0]].values.size();
    l1_total += r1;
    if (stop) continue;
    std::atomic<size_t> next{0};
    std::atomic<u64> ev{0}, lf{0}, done{0};
    std::atomic<bool> halt{false};
    // level-1 positions in a strided order (stride coprime to r1) so that a bounded sample
    // spans the whole range instead of its first values
    size_t stride = r1 > 1 ? (size_t)(2654435761ull % r1) : 1;
    if (stride == 0) stride = 1;
    while (r1 > 1 && std::gcd(stride, r1) != 1) stride++;
    auto worker = [&]() {
      GroupRun gr;
      gr.s = &s;
      gr.members = members;
      u64 mylf = 0;
      gr.sink = [&mylf](const i64*) { mylf++; };
      for (;;) {
        if (halt.load()) break;
        size_t j = next.fetch_add(1);
        if (j >= r1) break;
        j = (size_t)(((unsigned __int128)j * stride) % r1);
        gr.run(j, j + 1);
        u64 e = 0;
        for (auto& l : gr.lv) e += l.evals;
        ev += e;
        done++;
        double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        if (el > budget_s) halt = true;
      }
      lf += mylf;
    };
    std::vector<std::thread> th;
    for (int t = 0; t < std::max(1, threads); t++) th.emplace_back(worker);
    for (auto& t : th) t.join();
    evals += ev;
    leaves += lf;
    l1_done += done;
    if (halt) stop = true;
  }
  double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  std::printf("{\"seconds\":%.6f,\"evals\":%" PRIu64 ",\"leaves\":%" PRIu64 ",\"level1_done\":%" PRIu64
              ",\"level1_total\":%" PRIu64 ",\"threads\":%d}\n",
              el, evals, leaves, l1_done, l1_total, threads);
  return 0;
}

int main(int argc, char** argv) {
  if (argc < 3) {
    std::fprintf(stderr,
                 "usage: atf_oracle info|o1|leaves|decode|check|time|width SPEC.json [args] [--threads T] "
                 "[--native c1|c2:N|c3:M,N,K|saxpy:N] [--native-check] [--hash] [--budget S]\n");
    return 2;
  }
  std::string cmd = argv[1];
  std::vector<std::string> pos;
  int threads = 1;
  bool want_hash = false;
  double budget = 10.0;
  for (int i = 2; i < argc; i++) {
    std::string a = argv[i];
    if (a == "--threads") threads = std::atoi(argv[++i]);
    else if (a == "--native") g_native = make_native(argv[++i]);
    else if (a == "--native-check") g_native_check = true;
    else if (a == "--hash") want_hash = true;
    else if (a == "--budget") budget = std::atof(argv[++i]);
    else pos.push_back(a);
  }
  if (g_native_check && !g_native) { std::fprintf(stderr, "--native-check needs --native\n"); return 2; }
  try {
    Spec s = load_spec(pos.at(0));
    if (cmd == "info") return cmd_info(s, threads, want_hash);
    if (cmd == "width") return std::printf("{\"w64\":%s}\n", g_w64 ? "true" : "false"), 0;
    if (cmd == "o1") return cmd_o1(s, pos.size() > 1 ? pos[1].c_str() : nullptr);
    if (cmd == "leaves") return cmd_leaves(s, std::atoi(pos.at(1).c_str()), pos.at(2).c_str());
    if (cmd == "decode") return cmd_decode(s, pos.at(1).c_str(), pos.at(2).c_str(), threads);
    if (cmd == "check") return cmd_check(s, pos.at(1).c_str(), pos.size() > 2 ? pos.at(2).c_str() : nullptr);
    if (cmd == "time") return cmd_time(s, threads, budget);
    std::fprintf(stderr, "unknown command %s\n", cmd.c_str());
    return 2;
  } catch (std::exception& e) {
    std::printf("{\"error\":\"%s\"}\n", e.what());
    return 3;
  }
}
