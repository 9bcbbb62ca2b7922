// kernels.cu — sm_100a kernels of the ATF search-space generator.
//
// expand_kernel: one launch = one tree level of one parameter group.  It fuses the
// three steps of SURVEY.md §8(a) A4-A6 into a single pass:
//   count  — every (frontier node, candidate value) pair is evaluated against the
//            level parameter's constraint ("values for which the constraint
//            returns false are filtered out of the range"; ATF "filters out
//            invalid configurations by iterating over the constrained ranges");
//   scan   — a block scan of the per-warp accept counts plus a decoupled look-back
//            across tiles gives every accepted pair its global child index and every
//            frontier node its CSR first-child offset;
//   emit   — accepted pairs write the child's packed path record (parent record with
//            the candidate's range position inserted) with coalesced vector stores.
// Tiles are taken in ticket order by persistent CTAs, so every tile's predecessors
// are running or done (forward progress of the look-back).
//
// Candidate values and their divisibility magics live in registers (each thread
// owns CPT candidates for the whole launch); node-invariant operands (hoisted by
// the host planner) live in shared memory, one set per frontier node of the tile.
#include <cuda_runtime.h>
#include <cuda/atomic>
#include <stdint.h>

#include "atf_internal.hpp"

namespace atf {

#define FULL 0xffffffffu

// ---------------------------------------------------------------- generic interpreter
// Semantics of SURVEY.md §8(b) (same as the C ABI doc in include/atfgen.h); int64
// stack, poison on a zero divisor; strict evaluation.
__device__ __forceinline__ int64_t run_code(const int32_t* code, int len, int64_t x, const int64_t* slots,
                                            int stride, bool& poison) {
  int64_t st[kMaxStack];
  int sp = 0;
  for (int i = 0; i < len;) {
    const int op = code[i];
    if (op == 1) { st[sp++] = x; i += 1; continue; }
    if (op == OP_SLOT) { st[sp++] = slots[(int64_t)code[i + 1] * stride]; i += 2; continue; }
    if (op == 3) {
      st[sp++] = (int64_t)(((uint64_t)(uint32_t)code[i + 2] << 32) | (uint64_t)(uint32_t)code[i + 1]);
      i += 3;
      continue;
    }
    if (op == 21) { st[sp - 1] = (st[sp - 1] == 0); i += 1; continue; }
    const int64_t b = st[--sp];
    const int64_t a = st[sp - 1];
    int64_t r = 0;
    switch (op) {
      case 4: r = (int64_t)((uint64_t)a + (uint64_t)b); break;
      case 5: r = (int64_t)((uint64_t)a - (uint64_t)b); break;
      case 6: r = (int64_t)((uint64_t)a * (uint64_t)b); break;
      case 7: if (b == 0) { poison = true; r = 0; } else if (b == -1) { r = (int64_t)(0ull - (uint64_t)a); } else { r = a / b; } break;
      case 8: if (b == 0) { poison = true; r = 0; } else if (b == -1) { r = 0; } else { r = a % b; } break;
      case 9: r = a < b ? a : b; break;
      case 10: r = a > b ? a : b; break;
      case 11: r = (a == b); break;
      case 12: r = (a != b); break;
      case 13: r = (a < b); break;
      case 14: r = (a <= b); break;
      case 15: r = (a > b); break;
      case 16: r = (a >= b); break;
      case 17: if (a == 0) { poison = true; r = 0; } else if (a == -1) { r = 1; } else { r = (b % a == 0); } break;
      case 18: if (b == 0) { poison = true; r = 0; } else if (b == -1) { r = 1; } else { r = (a % b == 0); } break;
      case 19: r = (a != 0) & (b != 0); break;
      case 20: r = (a != 0) | (b != 0); break;
      default: poison = true; break;
    }
    st[sp - 1] = r;
    i += 1;
  }
  return sp == 1 ? st[0] : (poison = true, 0);
}

__device__ __forceinline__ uint64_t uabs64(int64_t v) { return v < 0 ? 0ull - (uint64_t)v : (uint64_t)v; }

__device__ __forceinline__ bool rel_holds(int rel, int64_t l, int64_t r) {
  switch (rel) {
    case R_EQ: return l == r;
    case R_NE: return l != r;
    case R_LT: return l < r;
    case R_LE: return l <= r;
    case R_GT: return l > r;
    default: return l >= r;
  }
}
__device__ __forceinline__ bool rel_holds32(int rel, int32_t l, int32_t r) {
  switch (rel) {
    case R_EQ: return l == r;
    case R_NE: return l != r;
    case R_LT: return l < r;
    case R_LE: return l <= r;
    case R_GT: return l > r;
    default: return l >= r;
  }
}

// ---------------------------------------------------------------- look-back
// Tile status word: bits 63..62 = flag (0 none, 1 aggregate, 2 inclusive prefix),
// bits 61..0 = value.
constexpr unsigned long long kFlagA = 1ull << 62, kFlagP = 2ull << 62, kValMask = (1ull << 62) - 1;

__device__ __forceinline__ void status_store(unsigned long long* p, unsigned long long v) {
  cuda::atomic_ref<unsigned long long, cuda::thread_scope_device> ref(*p);
  ref.store(v, cuda::memory_order_relaxed);
}
__device__ __forceinline__ unsigned long long status_load(unsigned long long* p) {
  cuda::atomic_ref<unsigned long long, cuda::thread_scope_device> ref(*p);
  return ref.load(cuda::memory_order_relaxed);
}

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
  return v;
}

// Called by one full warp.  Returns the exclusive prefix of tile `tile`.
__device__ unsigned long long lookback(unsigned long long* status, uint64_t tile, unsigned long long agg,
                                       int lane) {
  if (tile == 0) {
    if (lane == 0) status_store(&status[0], kFlagP | agg);
    return 0;
  }
  if (lane == 0) status_store(&status[tile], kFlagA | agg);
  unsigned long long excl = 0;
  int64_t idx = (int64_t)tile - 1 - lane;
  for (;;) {
    unsigned long long st = idx >= 0 ? status_load(&status[idx]) : kFlagP;
    while (__any_sync(FULL, (st >> 62) == 0)) {
      if ((st >> 62) == 0) st = status_load(&status[idx]);
    }
    const unsigned pm = __ballot_sync(FULL, (st >> 62) == 2);
    unsigned long long v = st & kValMask;
    if (pm) {
      const int first = __ffs(pm) - 1;  // nearest predecessor with an inclusive prefix
      if (lane > first) v = 0;
      excl += warp_sum_u64(v);
      break;
    }
    excl += warp_sum_u64(v);
    idx -= 32;
  }
  if (lane == 0) status_store(&status[tile], kFlagP | (excl + agg));
  return excl;
}

// ---------------------------------------------------------------- expand kernel
template <int CPT>
struct Cands {
  int32_t x[CPT];
  uint32_t j[CPT];   // range position
  uint32_t ax[CPT];  // |x|
  uint32_t m32[CPT]; // ceil(2^32 / |x|)  (0 for |x| in {0, 1}: 1 wraps)
  uint64_t m64[CPT]; // ceil(2^64 / |x|)
  bool v[CPT];       // owned and inside the range
};

template <int W>
__device__ __forceinline__ void store_record(uint32_t* dst, const uint32_t* rec) {
  if constexpr (W == 1) {
    dst[0] = rec[0];
  } else if constexpr (W == 2) {
    *reinterpret_cast<uint2*>(dst) = make_uint2(rec[0], rec[1]);
  } else if constexpr (W == 4) {
    *reinterpret_cast<uint4*>(dst) = make_uint4(rec[0], rec[1], rec[2], rec[3]);
  } else {
    *reinterpret_cast<uint4*>(dst) = make_uint4(rec[0], rec[1], rec[2], rec[3]);
    *reinterpret_cast<uint4*>(dst + 4) = make_uint4(rec[4], rec[5], rec[6], rec[7]);
  }
}

template <int W>
__device__ __forceinline__ void load_record(const uint32_t* src, uint32_t* rec) {
  if constexpr (W == 1) {
    rec[0] = __ldg(src);
  } else if constexpr (W == 2) {
    const uint2 v = __ldg(reinterpret_cast<const uint2*>(src));
    rec[0] = v.x; rec[1] = v.y;
  } else {
#pragma unroll
    for (int q = 0; q < W / 4; q++) {
      const uint4 v = __ldg(reinterpret_cast<const uint4*>(src) + q);
      rec[4 * q] = v.x; rec[4 * q + 1] = v.y; rec[4 * q + 2] = v.z; rec[4 * q + 3] = v.w;
    }
  }
}

// Per-node prologue: unpack ancestor values, evaluate hoisted invariants, gates and
// per-term operands into shared memory (node `i` of the tile, global index gnode).
template <int W>
__device__ void prologue_node(const LevelArgs& a, uint64_t gnode, int i, uint32_t* s_ok, uint32_t* s_rec,
                              int64_t* s_opa, int64_t* s_opb, int64_t* s_slots) {
  const int tn = a.tile_nodes;
  uint32_t rec[W];
  if (a.level == 0) {
#pragma unroll
    for (int w = 0; w < W; w++) rec[w] = 0;
  } else {
    load_record<W>(a.parent_rec + gnode * W, rec);
  }
#pragma unroll
  for (int w = 0; w < W; w++) s_rec[i * W + w] = rec[w];
  int64_t slots[kMaxSlots];
  for (int s = 0; s < a.n_pv; s++) {
    uint32_t word = 0;
#pragma unroll
    for (int w = 0; w < W; w++)
      if (w == a.pv_word[s]) word = rec[w];
    const uint32_t bits = (uint32_t)a.pv_bits[s];
    const uint32_t pos = bits ? (word >> a.pv_shift[s]) & ((bits >= 32) ? 0xffffffffu : ((1u << bits) - 1u)) : 0u;
    slots[s] = a.pv_range[s][pos];
  }
  bool poison = false;
  for (int s = a.n_pv; s < a.n_slots; s++)
    slots[s] = run_code(a.code + a.inv_off[s], a.inv_len[s], 0, slots, 1, poison);
  bool ok = !poison;
  for (int g = 0; g < a.n_gates; g++) ok = ok && (slots[a.gate_slot[g]] != 0);
  for (int t = 0; t < a.n_terms; t++) {
    const Term& T = a.terms[t];
    int64_t A = 0, B = 0;
    switch (T.kind) {
      case T_CMP: A = slots[T.slot_a]; B = slots[T.slot_b]; break;
      case T_DIVX: A = (int64_t)uabs64(slots[T.slot_a]); break;
      case T_MULX: {
        const uint64_t d = uabs64(slots[T.slot_a]);
        if (d == 0) ok = false;
        A = (int64_t)d;
        if (T.variant == V16) B = d ? (int64_t)(0xffffffffu / (uint32_t)d + 1u) : 0;
        else if (T.variant == V32) B = d ? (int64_t)(~0ull / d + 1ull) : 0;
        break;
      }
      case T_DIVPROD: {
        const uint64_t av = uabs64(slots[T.slot_a]), bv = uabs64(slots[T.slot_b]);
        if (av == 0) { ok = false; A = 0; }
        else if (bv % av != 0) { ok = false; A = 0; }
        else A = (int64_t)(bv / av);
        break;
      }
      case T_QDIV: A = (int64_t)uabs64(slots[T.slot_a]); B = (int64_t)uabs64(slots[T.slot_b]); break;
      default: break;
    }
    s_opa[t * tn + i] = A;
    s_opb[t * tn + i] = B;
  }
  if (s_slots)
    for (int s = 0; s < a.n_slots; s++) s_slots[s * tn + i] = slots[s];
  s_ok[i] = ok ? 1u : 0u;
}

// Evaluate term T for all (pass, candidate) items of this thread; returns accept bits
// (bit p*CPT + c).  Only bits set in `acc` matter.
template <int CPT>
__device__ __forceinline__ uint32_t eval_term(const LevelArgs& a, const Term& T, int t, const Cands<CPT>& cd,
                                              uint32_t acc, int n_off, int tn, int tn_valid, const int64_t* s_opa,
                                              const int64_t* s_opb, const int64_t* s_slots, const uint32_t* s_q,
                                              bool skip_empty_passes) {
  uint32_t bits = 0;
  const int np = a.np, npp = a.npp;
  const int64_t* opa = s_opa + t * tn;
  const int64_t* opb = s_opb + t * tn;
  for (int p = 0; p < np; p++) {
    const int nl = p * npp + n_off;
    const uint32_t pm = ((1u << CPT) - 1u) << (p * CPT);
    if (skip_empty_passes && !__any_sync(FULL, acc & pm)) continue;
    if (nl >= tn_valid) continue;
    uint32_t pb = 0;
    switch (T.kind) {
      case T_DIVX:
      case T_DIVPROD: {
        const uint64_t n = (uint64_t)opa[nl];
        if (T.variant == V16) {
          const uint32_t n32 = (uint32_t)n;
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)((n32 * cd.m32[c] <= cd.m32[c] - 1u) & (cd.ax[c] != 0)) << c;
        } else if (T.variant == V32) {
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)((n * cd.m64[c] <= cd.m64[c] - 1ull) & (cd.ax[c] != 0)) << c;
        } else {
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)(cd.ax[c] != 0 && n % cd.ax[c] == 0) << c;
        }
        break;
      }
      case T_MULX: {
        const uint64_t d = (uint64_t)opa[nl];
        const uint64_t md = (uint64_t)opb[nl];
        if (T.variant == V16) {
          const uint32_t m = (uint32_t)md;
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)(cd.ax[c] * m <= m - 1u) << c;
        } else if (T.variant == V32) {
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)((uint64_t)cd.ax[c] * md <= md - 1ull) << c;
        } else {
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)(d != 0 && (uint64_t)cd.ax[c] % d == 0) << c;
        }
        break;
      }
      case T_QDIV: {
        const uint64_t num = (uint64_t)opa[nl], nb = (uint64_t)opb[nl];
        if (T.variant == V16) {
          const uint32_t num32 = (uint32_t)num, nb32 = (uint32_t)nb;
#pragma unroll
          for (int c = 0; c < CPT; c++) {
            const uint32_t q = cd.ax[c] == 1 ? num32 : __umulhi(num32, cd.m32[c]);
            bool ok;
            if (T.use_qtable) {
              const uint32_t mq = s_q[q];
              ok = (nb32 * mq <= mq - 1u);
            } else {
              ok = q != 0 && nb32 % (q ? q : 1u) == 0;
            }
            pb |= (uint32_t)(ok & (q != 0) & (cd.ax[c] != 0)) << c;
          }
        } else if (T.variant == V32) {
#pragma unroll
          for (int c = 0; c < CPT; c++) {
            const uint64_t q = cd.ax[c] == 1 ? num : __umul64hi(cd.m64[c], num);
            pb |= (uint32_t)(cd.ax[c] != 0 && q != 0 && nb % (q ? q : 1ull) == 0) << c;
          }
        } else {
#pragma unroll
          for (int c = 0; c < CPT; c++) {
            const uint64_t q = cd.ax[c] ? num / cd.ax[c] : 0;
            pb |= (uint32_t)(cd.ax[c] != 0 && q != 0 && nb % (q ? q : 1ull) == 0) << c;
          }
        }
        break;
      }
      case T_CMP: {
        const int64_t A = opa[nl], B = opb[nl];
        if (T.variant == V32) {
          const int32_t A32 = (int32_t)A, B32 = (int32_t)B;
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)rel_holds32(T.rel, A32 * cd.x[c], B32) << c;
        } else {
#pragma unroll
          for (int c = 0; c < CPT; c++) pb |= (uint32_t)rel_holds(T.rel, A * (int64_t)cd.x[c], B) << c;
        }
        break;
      }
      default: {  // T_GENERIC: interpret the conjunct per candidate
#pragma unroll
        for (int c = 0; c < CPT; c++) {
          if (!((acc >> (p * CPT + c)) & 1u)) continue;
          bool poison = false;
          const int64_t v = run_code(a.code + T.code_off, T.code_len, cd.x[c], s_slots + nl, tn, poison);
          pb |= (uint32_t)(!poison && v != 0) << c;
        }
        break;
      }
    }
    bits |= pb << (p * CPT);
  }
  return bits;
}

template <int W, int CPT>
__global__ void __launch_bounds__(1024) expand_kernel(const __grid_constant__ LevelArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  const SmemLayout L = expand_layout(a, W);
  uint32_t* ctl = reinterpret_cast<uint32_t*>(smem + L.ctl);
  uint32_t* s_ok = reinterpret_cast<uint32_t*>(smem + L.ok);
  uint32_t* s_rec = reinterpret_cast<uint32_t*>(smem + L.rec);
  int64_t* s_opa = reinterpret_cast<int64_t*>(smem + L.opa);
  int64_t* s_opb = reinterpret_cast<int64_t*>(smem + L.opb);
  int64_t* s_slots = L.slots >= 0 ? reinterpret_cast<int64_t*>(smem + L.slots) : nullptr;
  uint32_t* s_wcnt = reinterpret_cast<uint32_t*>(smem + L.wcnt);
  uint32_t* s_wtot = reinterpret_cast<uint32_t*>(smem + L.wtot);
  uint32_t* s_q = L.qtab >= 0 ? reinterpret_cast<uint32_t*>(smem + L.qtab) : nullptr;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int B = blockDim.x, NW = B >> 5;
  const int r = a.r;

  if (s_q)
    for (uint32_t q = tid; q <= a.qmax; q += B) s_q[q] = q ? (0xffffffffu / q + 1u) : 0u;

  // thread -> (node offset within a pass, owned candidates)
  int n_off;
  bool tactive;
  if (CPT == 1) {
    n_off = tid / r;
    tactive = n_off < a.npp;
  } else {
    n_off = 0;
    tactive = true;
  }
  Cands<CPT> cd;
  auto load_cands = [&](int64_t chunk) {
#pragma unroll
    for (int c = 0; c < CPT; c++) {
      int64_t j = CPT == 1 ? (int64_t)(tid % r) + chunk * B : chunk * (int64_t)B * CPT + (int64_t)c * B + tid;
      const bool v = tactive && j < r;
      const int32_t x = v ? __ldg(a.cand + j) : 0;
      const uint32_t ax = x < 0 ? 0u - (uint32_t)x : (uint32_t)x;
      cd.x[c] = x;
      cd.j[c] = (uint32_t)j;
      cd.ax[c] = ax;
      cd.m32[c] = ax ? 0xffffffffu / ax + 1u : 0u;
      cd.m64[c] = (a.need_m64 && ax) ? ~0ull / ax + 1ull : 0ull;
      cd.v[c] = v;
    }
  };
  if (a.n_chunks == 1) load_cands(0);
  const int items = a.np * CPT;

  for (;;) {
    if (tid == 0) ctl[0] = atomicAdd(a.tile_counter, 1u);
    __syncthreads();
    const uint64_t tile = ctl[0];
    if (tile >= a.n_tiles) break;
    uint64_t node0;
    int64_t chunk = 0;
    int tn;
    if (a.n_chunks == 1) {
      node0 = tile * (uint64_t)a.tile_nodes;
      const uint64_t rem = a.n_parents - node0;
      tn = rem < (uint64_t)a.tile_nodes ? (int)rem : a.tile_nodes;
    } else {
      node0 = tile / (uint64_t)a.n_chunks;
      chunk = (int64_t)(tile % (uint64_t)a.n_chunks);
      tn = 1;
      load_cands(chunk);
    }
    // ---- prologue: one thread per frontier node of the tile
    for (int i = tid; i < tn; i += B) prologue_node<W>(a, node0 + i, i, s_ok, s_rec, s_opa, s_opb, s_slots);
    __syncthreads();

    // ---- count: evaluate the level's conjunction
    uint32_t acc = 0;
    for (int p = 0; p < a.np; p++) {
      const int nl = p * a.npp + n_off;
      if (!tactive || nl >= tn || !s_ok[nl]) continue;
#pragma unroll
      for (int c = 0; c < CPT; c++)
        if (cd.v[c]) acc |= 1u << (p * CPT + c);
    }
    for (int t = 0; t < a.n_terms; t++) {
      if (!__any_sync(FULL, acc)) break;  // top-level AND: a rejected item stays rejected
      acc &= eval_term<CPT>(a, a.terms[t], t, cd, acc, n_off, a.tile_nodes, tn, s_opa, s_opb, s_slots, s_q, t > 0);
    }

    // ---- scan: per-warp counts in item order (pass, cand-slot, warp), block scan, look-back
    for (int k = 0; k < items; k++) {
      const unsigned bal = __ballot_sync(FULL, (acc >> k) & 1u);
      if (lane == 0) s_wcnt[k * NW + warp] = __popc(bal);
    }
    __syncthreads();
    const int n_items = items * NW;
    {
      uint32_t v = tid < n_items ? s_wcnt[tid] : 0u;
      uint32_t incl = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
      }
      if (lane == 31) s_wtot[warp] = incl;
      __syncthreads();
      if (warp == 0) {
        uint32_t wt = lane < NW ? s_wtot[lane] : 0u;
        uint32_t wi = wt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(FULL, wi, o);
          if (lane >= o) wi += y;
        }
        if (lane < NW) s_wtot[lane] = wi - wt;  // exclusive warp offsets
        if (lane == 31) s_wtot[32] = wi;        // tile total
      }
      __syncthreads();
      if (tid < n_items) s_wcnt[tid] = incl - v + s_wtot[warp];
    }
    if (warp == 0) {
      const unsigned long long total = s_wtot[32];
      const unsigned long long base = lookback(a.status, tile, total, lane);
      if (lane == 0) {
        ctl[2] = (uint32_t)base;
        ctl[3] = (uint32_t)(base >> 32);
        if (tile == a.n_tiles - 1) {
          *a.total_out = base + total;
          a.csr[a.n_parents] = base + total;
        }
      }
    }
    __syncthreads();
    const uint64_t base = (uint64_t)ctl[2] | ((uint64_t)ctl[3] << 32);

    // ---- emit: CSR offsets of the tile's nodes and the accepted children's records
    const unsigned lt = (1u << lane) - 1u;
    for (int k = 0; k < items; k++) {
      const int p = k / CPT, c = k % CPT;
      const bool b = (acc >> k) & 1u;
      const unsigned bal = __ballot_sync(FULL, b);
      const int nl = p * a.npp + n_off;
      const uint64_t rank = base + s_wcnt[k * NW + warp] + __popc(bal & lt);
      const bool first = CPT == 1 ? (tactive && cd.j[0] == 0) : (c == 0 && tid == 0 && chunk == 0);
      if (first && nl < tn) a.csr[node0 + nl] = rank;
      if (b) {
        if (rank < a.child_cap) {
          uint32_t rec[W];
#pragma unroll
          for (int w = 0; w < W; w++) rec[w] = s_rec[nl * W + w];
#pragma unroll
          for (int w = 0; w < W; w++)
            if (w == a.field_word) rec[w] |= cd.j[c] << a.field_shift;
          store_record<W>(a.child_rec + rank * W, rec);
        } else {
          atomicOr(a.overflow_flag, 1u);
        }
      }
    }
    __syncthreads();
  }
}

template <int W, int CPT>
static int launch_wc(const LevelArgs& a, void* stream) {
  auto k = expand_kernel<W, CPT>;
  const int smem = expand_layout(a, W).total;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return (int)e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, a.block, smem);
  if (e != cudaSuccess) return (int)e;
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (per_sm < 1) per_sm = 1;
  uint64_t grid = (uint64_t)sms * per_sm;
  if (grid > a.n_tiles) grid = a.n_tiles;
  if (grid < 1) grid = 1;
  k<<<(unsigned)grid, a.block, smem, (cudaStream_t)stream>>>(a);
  return (int)cudaGetLastError();
}

template <int W>
static int launch_w(const LevelArgs& a, void* stream) {
  switch (a.cpt) {
    case 1: return launch_wc<W, 1>(a, stream);
    case 2: return launch_wc<W, 2>(a, stream);
    case 4: return launch_wc<W, 4>(a, stream);
    case 8: return launch_wc<W, 8>(a, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

int launch_expand(const LevelArgs& a, int words, void* stream) {
  switch (words) {
    case 1: return launch_w<1>(a, stream);
    case 2: return launch_w<2>(a, stream);
    case 4: return launch_w<4>(a, stream);
    case 8: return launch_w<8>(a, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

int expand_smem_bytes(const LevelArgs& a, int words) { return expand_layout(a, words).total; }

// ---------------------------------------------------------------- decode
// index -> mixed-radix digits (group 0 most significant, P:229-231 reading #11) ->
// per group: leaf record -> positions -> values; int32 SoA output.
__global__ void decode_kernel(const __grid_constant__ DecodeArgs a, const uint64_t* __restrict__ idx,
                              const uint64_t* __restrict__ digits, int64_t n, int32_t* __restrict__ out,
                              int64_t ld, unsigned int* bad, uint64_t S, int s_fits) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    bool valid = true;
    uint64_t rem = 0;
    if (idx) {
      rem = __ldg(idx + i);
      valid = s_fits && rem < S;
    } else {
      for (int g = 0; g < a.n_groups; g++) valid = valid && __ldg(digits + (int64_t)g * n + i) < a.gsize[g];
    }
    if (!valid) {
      for (int p = 0; p < a.n_params; p++) out[(int64_t)p * ld + i] = INT32_MIN;
      atomicOr(bad, 1u);
      continue;
    }
    for (int g = a.n_groups - 1; g >= 0; g--) {
      uint64_t d;
      if (idx) {
        const uint64_t sz = a.gsize[g];
        d = rem % sz;
        rem /= sz;
      } else {
        d = __ldg(digits + (int64_t)g * n + i);
      }
      const int W = a.words[g];
      const uint32_t* rp = a.leaves[g] + d * (uint64_t)W;
      uint32_t rec[8];
      if (W == 1) {
        rec[0] = __ldg(rp);
      } else if (W == 2) {
        const uint2 v = __ldg(reinterpret_cast<const uint2*>(rp));
        rec[0] = v.x; rec[1] = v.y;
      } else {
        for (int q = 0; q < W / 4; q++) {
          const uint4 v = __ldg(reinterpret_cast<const uint4*>(rp) + q);
          rec[4 * q] = v.x; rec[4 * q + 1] = v.y; rec[4 * q + 2] = v.z; rec[4 * q + 3] = v.w;
        }
      }
      for (int l = a.lvl_begin[g]; l < a.lvl_begin[g + 1]; l++) {
        const uint32_t bits = (uint32_t)a.lvl_bits[l];
        const uint32_t pos = bits ? (rec[a.lvl_word[l]] >> a.lvl_shift[l]) & ((1u << bits) - 1u) : 0u;
        out[(int64_t)a.lvl_param[l] * ld + i] = __ldg(a.lvl_range[l] + pos);
      }
    }
  }
}

static int launch_decode(const DecodeArgs& a, const uint64_t* idx, const uint64_t* digits, int64_t n, int32_t* out,
                         int64_t ld, unsigned int* bad, void* stream) {
  if (n <= 0) return 0;
  uint64_t S = 1;
  int fits = 1;
  for (int g = 0; g < a.n_groups; g++) {
    const unsigned __int128 t = (unsigned __int128)S * a.gsize[g];
    if (t >> 64) fits = 0;
    S = (uint64_t)t;
  }
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int64_t blocks = (n + 255) / 256;
  const int64_t cap = (int64_t)sms * 8;
  if (blocks > cap) blocks = cap;
  decode_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(a, idx, digits, n, out, ld, bad, S, fits);
  return (int)cudaGetLastError();
}

int launch_decode_indices(const DecodeArgs& a, const uint64_t* idx, int64_t n, int32_t* out, int64_t ld,
                          unsigned int* bad, void* stream) {
  return launch_decode(a, idx, nullptr, n, out, ld, bad, stream);
}
int launch_decode_digits(const DecodeArgs& a, const uint64_t* digits, int64_t n, int32_t* out, int64_t ld,
                         unsigned int* bad, void* stream) {
  return launch_decode(a, nullptr, digits, n, out, ld, bad, stream);
}

// ---------------------------------------------------------------- standalone scan (tests)
// Exclusive scan u32 -> u64 with the same look-back as expand_kernel; out[n] = total.
__global__ void scan_kernel(const uint32_t* __restrict__ in, uint64_t* __restrict__ out, int64_t n,
                            unsigned long long* status, unsigned int* counter, uint64_t n_tiles) {
  __shared__ uint32_t s_tile;
  __shared__ unsigned long long s_wt[33];
  __shared__ unsigned long long s_base;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int ITEMS = 4;
  for (;;) {
    if (tid == 0) s_tile = atomicAdd(counter, 1u);
    __syncthreads();
    const uint64_t tile = s_tile;
    if (tile >= n_tiles) break;
    const int64_t i0 = (int64_t)tile * blockDim.x * ITEMS + (int64_t)tid * ITEMS;
    unsigned long long v[ITEMS], sum = 0;
    for (int q = 0; q < ITEMS; q++) {
      v[q] = (i0 + q < n) ? in[i0 + q] : 0u;
      sum += v[q];
    }
    unsigned long long incl = sum;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(FULL, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) s_wt[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      const int NW = blockDim.x >> 5;
      unsigned long long wt = lane < NW ? s_wt[lane] : 0ull, wi = wt;
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(FULL, wi, o);
        if (lane >= o) wi += y;
      }
      if (lane < NW) s_wt[lane] = wi - wt;
      const unsigned long long tot = __shfl_sync(FULL, wi, 31);
      const unsigned long long base = lookback(status, tile, tot, lane);
      if (lane == 0) {
        s_base = base;
        if (tile == n_tiles - 1) out[n] = base + tot;
      }
    }
    __syncthreads();
    unsigned long long run = s_base + s_wt[warp] + incl - sum;
    for (int q = 0; q < ITEMS; q++) {
      if (i0 + q < n) out[i0 + q] = run;
      run += v[q];
    }
    __syncthreads();
  }
}

int launch_scan_u32(const uint32_t* in, uint64_t* out, int64_t n, unsigned long long* status, unsigned int* counter,
                    void* stream) {
  const int B = 256;
  const uint64_t n_tiles = n > 0 ? (uint64_t)((n + B * 4 - 1) / (B * 4)) : 1;
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint64_t grid = (uint64_t)sms * 4;
  if (grid > n_tiles) grid = n_tiles;
  scan_kernel<<<(unsigned)grid, B, 0, (cudaStream_t)stream>>>(in, out, n, status, counter, n_tiles);
  return (int)cudaGetLastError();
}

__global__ void add_offset_kernel(uint64_t* data, uint64_t n, uint64_t add) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    data[i] += add;
}
int launch_add_offset(uint64_t* data, uint64_t n, uint64_t add, void* stream) {
  if (n == 0) return 0;
  uint64_t blocks = (n + 255) / 256;
  if (blocks > 4096) blocks = 4096;
  add_offset_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(data, n, add);
  return (int)cudaGetLastError();
}

}  // namespace atf
