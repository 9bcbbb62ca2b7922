// expand.cuh — the level-expansion kernels (SURVEY.md §8(a) A4-A6 fused: count, scan,
// emit), instantiated per record width W in expand_w{1,2,4,8}.cu.
#pragma once
#include <type_traits>

#include "dev_common.cuh"

namespace atf {

// ---------------------------------------------------------------- exact term evaluation
// One (frontier node, candidate) pair against conjunct T (SURVEY.md §8(b) semantics; the
// planner's atoms are exact rewrites of the bytecode).  A, Bv: the
// node's operands of T (prologue); x: candidate value, ax = |x|, m32 = ceil(2^32/ax)
// (0 for ax <= 1).  slots/stride: the node's slot column (generic terms only).
// X64: the level may be an int64 parameter's (reading #22): a generic term maps the candidate
// position x to its int64 value.  Hot-filter levels never are (their callers pass false and keep
// the code of the int32 path).
template <bool X64>
__device__ __forceinline__ bool term_accepts(const LevelArgs& a, const Term& T, int64_t A, int64_t Bv, int32_t x,
                                             uint32_t ax, uint32_t m32, const uint32_t* s_q, const int64_t* slots,
                                             int stride) {
  switch (T.kind) {
    case T_DIVX:
    case T_DIVPROD: {  // x | n   (n = A = |m| or |b/a|); x == 0 -> poison -> reject
      if (ax == 0) return false;
      const uint64_t n = (uint64_t)A;
      if (T.variant == V16) return (uint32_t)n * m32 <= m32 - 1u;
      if (T.variant == V32) {
        const uint64_t m64 = udiv64f(~0ull, ax) + 1ull;
        return n * m64 <= m64 - 1ull;
      }
      return umod64f(n, ax) == 0;
    }
    case T_MULX: {  // d | x  (d = A != 0 checked by the node gate, Bv = magic(d))
      const uint64_t d = (uint64_t)A, md = (uint64_t)Bv;
      if (T.variant == V16) return ax * (uint32_t)md <= (uint32_t)md - 1u;
      if (T.variant == V32) return (uint64_t)ax * md <= md - 1ull;
      return d != 0 && umod64f(ax, d) == 0;
    }
    case T_QDIV: {  // (num / x) | nb; x == 0 or quotient 0 -> poison -> reject
      if (ax == 0) return false;
      const uint64_t num = (uint64_t)A, nb = (uint64_t)Bv;
      if (T.variant == V16) {
        const uint32_t q = ax == 1 ? (uint32_t)num : __umulhi((uint32_t)num, m32);
        if (q == 0) return false;
        if (T.use_qtable) {
          const uint32_t mq = s_q[q];
          return (uint32_t)nb * mq <= mq - 1u;
        }
        return divisible16((uint32_t)nb, q);
      }
      const uint64_t q = udiv64f(num, ax);
      return q != 0 && umod64f(nb, q) == 0;
    }
    case T_CMP:
      if (T.variant == V32) return rel_holds32(T.rel, (int32_t)A * x, (int32_t)Bv);
      return rel_holds(T.rel, A * (int64_t)x, Bv);
    default: {  // T_GENERIC: interpret the conjunct (int64 parameter: x is the position, reading #22)
      bool poison = false;
      const int64_t xv = (X64 && a.cand64) ? __ldg(a.cand64 + x) : (int64_t)x;
      const int64_t v = run_code(a.code + T.code_off, T.code_len, xv, slots, stride, poison);
      return !poison && v != 0;
    }
  }
}

// Narrow kernel: conjunct T over all r <= 64 candidates of one node, restricted to the
// candidates still set in m.  The kind/variant dispatch is hoisted out of the candidate
// loop; the 16-bit divisibility atoms are evaluated branch-free for every candidate.
__device__ __forceinline__ uint64_t term_mask_narrow(const LevelArgs& a, const Term& T, int64_t A, int64_t Bv,
                                                     uint64_t m, int r, const int32_t* s_cx, const uint32_t* s_cm,
                                                     const uint32_t* s_q, const int64_t* slots, int stride) {
  if ((T.kind == T_DIVX || T.kind == T_DIVPROD) && T.variant == V16) {
    // x | n  iff  n * magic(x) mod 2^32 < 2^16 (magic(0) = 2^16 excludes x == 0)
    const uint32_t n = (uint32_t)A;
    uint32_t lo = 0, hi = 0;
    for (int c = 0; c < r; c++) {
      const uint32_t mg = s_cm[c];
      const uint32_t ok = (uint32_t)((n * mg < 0x10000u) & (mg != 0x10000u));
      if (c < 32) lo |= ok << c; else hi |= ok << (c - 32);
    }
    return m & (((uint64_t)hi << 32) | lo);
  }
  if (T.kind == T_MULX && T.variant == V16) {
    const uint32_t md = (uint32_t)Bv, md1 = md - 1u;
    uint32_t lo = 0, hi = 0;
    for (int c = 0; c < r; c++) {
      const int32_t x = s_cx[c];
      const uint32_t ax = x < 0 ? 0u - (uint32_t)x : (uint32_t)x;
      const uint32_t ok = (uint32_t)(ax * md <= md1);
      if (c < 32) lo |= ok << c; else hi |= ok << (c - 32);
    }
    return m & (((uint64_t)hi << 32) | lo);
  }
  uint64_t out = 0, mm = m;
  while (mm) {
    const int c = __ffsll((long long)mm) - 1;
    mm &= mm - 1;
    const int32_t x = s_cx[c];
    const uint32_t ax = x < 0 ? 0u - (uint32_t)x : (uint32_t)x;
    if (term_accepts<true>(a, T, A, Bv, x, ax, s_cm[c], s_q, slots, stride)) out |= 1ull << c;
  }
  return out;
}

// Exact acceptance of candidate (x, m32) by node i of the tile (all conjuncts, node gate).
static __device__ __noinline__ bool node_accepts(const LevelArgs& a, int i, int tn, int32_t x, uint32_t m32,
                                             const uint32_t* s_ok, const int64_t* s_opa, const int64_t* s_opb,
                                             const int64_t* s_slots, const uint32_t* s_q) {
  if (!s_ok[i]) return false;
  const uint32_t ax = x < 0 ? 0u - (uint32_t)x : (uint32_t)x;
  for (int t = 0; t < a.n_terms; t++)
    if (!term_accepts<true>(a, a.terms[t], s_opa[t * tn + i], s_opb[t * tn + i], x, ax, m32, s_q,
                      s_slots ? s_slots + i : nullptr, tn))
      return false;
  return true;
}

// ---------------------------------------------------------------- records
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

// Per-node prologue: unpack ancestor values from the parent's path record, evaluate the
// hoisted node-invariant expressions, the node gates and every conjunct's operands into
// shared memory (node `i` of the tile, global index gnode).  Returns the gate result.
// X64: int64 ancestors possible (reading #22; never on hot-filter levels, see choose_geometry).
template <int W, bool X64 = true>
__device__ __forceinline__ bool prologue_node_impl(const LevelArgs& a, uint64_t gnode, int i, int tn, uint32_t* s_ok, uint32_t* s_rec,
                              int64_t* s_opa, int64_t* s_opb, int64_t* s_slots, bool rec_staged = false) {
  uint32_t rec[W];
  if (a.level == 0) {
#pragma unroll
    for (int w = 0; w < W; w++) rec[w] = 0;
  } else if (rec_staged) {  // the caller prefetched the record into s_rec
#pragma unroll
    for (int w = 0; w < W; w++) rec[w] = s_rec[i * W + w];
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
    slots[s] = (X64 && a.pv_range64[s]) ? a.pv_range64[s][pos] : (int64_t)a.pv_range[s][pos];
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
        else if (T.variant == V32) B = d ? (int64_t)(udiv64f(~0ull, d) + 1ull) : 0;
        break;
      }
      case T_DIVPROD: {
        const uint64_t av = uabs64(slots[T.slot_a]), bv = uabs64(slots[T.slot_b]);
        if (av == 0) { ok = false; A = 0; }
        else if (umod64f(bv, av) != 0) { ok = false; A = 0; }
        else A = (int64_t)udiv64f(bv, av);
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
  return ok;
}

// Out-of-line copy for the wide kernel (keeps the hot loop's registers free).
template <int W, bool X64>
__device__ __noinline__ bool prologue_node(const LevelArgs& a, uint64_t gnode, int i, int tn, uint32_t* s_ok,
                                           uint32_t* s_rec, int64_t* s_opa, int64_t* s_opb, int64_t* s_slots,
                                           bool rec_staged) {
  return prologue_node_impl<W, X64>(a, gnode, i, tn, s_ok, s_rec, s_opa, s_opb, s_slots, rec_staged);
}

// Block-wide exclusive scan of one u32 per thread (B <= 1024); returns the exclusive
// prefix, *total = block sum.  s_w: >= 33 u64 of shared scratch.  Ends with a barrier.
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t* total, unsigned long long* s_w) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, NW = blockDim.x >> 5;
  uint32_t incl = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) s_w[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const uint32_t wt = lane < NW ? (uint32_t)s_w[lane] : 0u;
    uint32_t wi = wt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL, wi, o);
      if (lane >= o) wi += y;
    }
    if (lane < NW) s_w[lane] = wi - wt;
    if (lane == 31) s_w[32] = wi;
  }
  __syncthreads();
  *total = (uint32_t)s_w[32];
  return incl - v + (uint32_t)s_w[warp];
}

// ---------------------------------------------------------------- narrow expand kernel
// One launch = one tree level of one group, for ranges of r <= 64 candidates.  Tile =
// blockDim.x * NPT frontier nodes; thread t owns the NPT consecutive nodes
// [t*NPT, t*NPT + NPT) of the tile (thread order = node order).  Per node: prologue ->
// exact term-major evaluation of the r candidates into a 64-bit accept mask (count, A4);
// per tile: block scan of the per-thread child counts (A5, tile part); every thread
// writes its nodes' tile-local CSR entries and its children records, in candidate order,
// into the tile's stash segment (emit, A6); scan_kernel + level_emit_kernel then place
// the segments.  The prologue's operand columns are per thread and reused node by node.
constexpr int kNarrowNPT = 4;

template <int W>
__global__ void __launch_bounds__(256) expand_narrow(const __grid_constant__ LevelArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  const SmemLayout L = expand_layout(a, W);
  uint32_t* ctl = reinterpret_cast<uint32_t*>(smem + L.ctl);
  uint32_t* s_ok = reinterpret_cast<uint32_t*>(smem + L.ok);
  uint32_t* s_rec = reinterpret_cast<uint32_t*>(smem + L.rec);
  int64_t* s_opa = reinterpret_cast<int64_t*>(smem + L.opa);
  int64_t* s_opb = reinterpret_cast<int64_t*>(smem + L.opb);
  int64_t* s_slots = L.slots >= 0 ? reinterpret_cast<int64_t*>(smem + L.slots) : nullptr;
  int32_t* s_cx = reinterpret_cast<int32_t*>(smem + L.cx);
  uint32_t* s_cm = reinterpret_cast<uint32_t*>(smem + L.cm);
  uint32_t* s_q = L.qtab >= 0 ? reinterpret_cast<uint32_t*>(smem + L.qtab) : nullptr;
  unsigned long long* s_w = reinterpret_cast<unsigned long long*>(smem + L.wtot);

  const int tid = threadIdx.x, lane = tid & 31, B = blockDim.x;
  const int r = a.r, tn_max = a.tile_nodes;  // = B * kNarrowNPT
  for (int j = tid; j < r; j += B) {
    s_cx[j] = __ldg(a.cand + j);
    s_cm[j] = __ldg(a.cand_magic + j);
  }
  if (s_q)
    for (uint32_t q = tid; q <= a.qmax; q += B) s_q[q] = q ? (0xffffffffu / q + 1u) : 0u;
  const uint64_t full = r >= 64 ? ~0ull : ((1ull << r) - 1ull);

  for (;;) {
    if (tid == 0) ctl[0] = atomicAdd(a.tile_counter, 1u);
    __syncthreads();
    const uint64_t tile = ctl[0];
    if (tile >= a.n_tiles) break;
    const uint64_t node0 = tile * (uint64_t)tn_max;
    const uint64_t rem = a.n_parents - node0;
    const int tn = rem < (uint64_t)tn_max ? (int)rem : tn_max;
    uint64_t mask[kNarrowNPT];
    uint32_t rec[kNarrowNPT][W];
    uint32_t cnt = 0;
#pragma unroll
    for (int k = 0; k < kNarrowNPT; k++) {
      const int i = tid * kNarrowNPT + k;
      mask[k] = 0;
      // the operand column of this thread (index tid) is reused for each of its nodes
      if (i < tn && prologue_node_impl<W>(a, node0 + i, tid, B, s_ok, s_rec, s_opa, s_opb, s_slots)) {
        uint64_t m = full;
        for (int t = 0; t < a.n_terms && m; t++)
          m = term_mask_narrow(a, a.terms[t], s_opa[t * B + tid], s_opb[t * B + tid], m, r, s_cx, s_cm, s_q,
                               s_slots ? s_slots + tid : nullptr, B);
        mask[k] = m;
      }
      if (i < tn) {
#pragma unroll
        for (int w = 0; w < W; w++) rec[k][w] = s_rec[tid * W + w];
      }
      cnt += (uint32_t)__popcll(mask[k]);
    }
    uint32_t total;
    const uint32_t excl = block_excl_scan(cnt, &total, s_w);
    // the tile's children go to a stash segment claimed with one atomic (no wait on other
    // tiles); scan_kernel + level_emit_kernel place the segments (as for wide levels)
    if (tid == 0) {
      const unsigned long long sg = total ? atomicAdd(a.stash_top, (unsigned long long)total) : 0ull;
      if (total && sg + total > a.stash_cap) atomicOr(a.overflow_flag, 1u);
      a.tile_total[tile] = total;
      a.tile_seg[tile] = sg;
      s_w[33] = sg;
    }
    __syncthreads();
    const uint64_t seg = s_w[33];
    uint32_t local = excl;  // tile-local child index (CSR gets it; the emit kernel adds the tile base)
#pragma unroll
    for (int k = 0; k < kNarrowNPT; k++) {
      const int i = tid * kNarrowNPT + k;
      if (i >= tn) break;
      a.csr[node0 + i] = local;
      uint64_t m = mask[k];
      while (m) {
        const int c = __ffsll((long long)m) - 1;
        m &= m - 1;
        const uint64_t rank = seg + local;
        if (rank < a.stash_cap) {
          uint32_t out[W];
#pragma unroll
          for (int w = 0; w < W; w++) out[w] = rec[k][w] | (w == a.field_word ? (uint32_t)c << a.field_shift : 0u);
          store_record<W>(a.stash + rank * W, out);
        }
        local++;
      }
    }
    __syncthreads();
  }
}

// Conjuncts other than the hot one, for the candidates still set in `mask` (bit c =
// candidate jg0 + c of the range).  Out of line: only reached on hot-filter survivors.
static __device__ __noinline__ uint32_t other_terms_mask(const LevelArgs& a, int i, int tn, int64_t jg0,
                                                        uint32_t mask, int skip, const int64_t* s_opa,
                                                        const int64_t* s_opb, const int64_t* s_slots,
                                                        const uint32_t* s_q) {
  for (int t = 0; t < a.n_terms && mask; t++) {
    if (t == skip) continue;
    const Term& T = a.terms[t];
    const int64_t A = s_opa[t * tn + i], Bv = s_opb[t * tn + i];
    uint32_t m = mask;
    if (T.kind == T_QDIV && T.variant == V16 && !T.use_qtable) {
      // (num / x) | nb, the 16-bit case hoisted out of the generic dispatch
      const uint32_t num = (uint32_t)A, nb = (uint32_t)Bv;
      while (m) {
        const int c = __ffs(m) - 1;
        m &= m - 1;
        const uint32_t ax = __ldg(a.cand_abs + jg0 + c);
        bool ok = false;
        if (ax != 0) {
          const uint32_t q = ax == 1 ? num : __umulhi(num, __ldg(a.cand_magic + jg0 + c));
          ok = q != 0 && divisible16(nb, q);
        }
        if (!ok) mask &= ~(1u << c);
      }
      continue;
    }
    if ((T.kind == T_DIVX || T.kind == T_DIVPROD) && T.variant == V16) {
      const uint32_t n = (uint32_t)A;
      while (m) {
        const int c = __ffs(m) - 1;
        m &= m - 1;
        const uint32_t mg = __ldg(a.cand_magic + jg0 + c);
        if (!(n * mg < 0x10000u && mg != 0x10000u)) mask &= ~(1u << c);
      }
      continue;
    }
    while (m) {
      const int c = __ffs(m) - 1;
      m &= m - 1;
      const int32_t x = __ldg(a.cand + jg0 + c);
      const uint32_t ax = x < 0 ? 0u - (uint32_t)x : (uint32_t)x;
      if (!term_accepts<false>(a, T, A, Bv, x, ax, __ldg(a.cand_magic + jg0 + c), s_q, s_slots ? s_slots + i : nullptr,
                               tn))
        mask &= ~(1u << c);
    }
  }
  return mask;
}

// Exact accept mask of node i over chunk candidates [jl0, jl0 + CPT), recorded in the
// node's bitmap, summary and count (shared-memory atomics, once per call).
template <int CPT, int HOT>
__device__ __forceinline__ void record_mask(const LevelArgs& a, int i, int tn, int jl0, int64_t j0,
                                            const uint32_t* s_ok, const uint32_t* s_hot, const uint32_t* s_hot2,
                                            const int64_t* s_opa, const int64_t* s_opb, const int64_t* s_slots,
                                            const uint32_t* s_q, uint32_t* s_bm, uint32_t* s_sum, uint32_t* s_cnt,
                                            int RW, int SW) {
  if (!s_ok[i]) return;
  const int64_t jg0 = j0 + jl0;
  uint32_t mask = 0;
  if (HOT == HOT_NONE) {
#pragma unroll
    for (int c = 0; c < CPT; c++)
      if (jg0 + c < a.r &&
          node_accepts(a, i, tn, __ldg(a.cand + jg0 + c), __ldg(a.cand_magic + jg0 + c), s_ok, s_opa, s_opb,
                       s_slots, s_q))
        mask |= 1u << c;
  } else {
    const uint32_t n = s_hot[i], d1 = s_hot2[i];
#pragma unroll
    for (int c = 0; c < CPT; c++) {
      if (jg0 + c < a.r) {
        bool ok;
        if (HOT == HOT_DIVX) {
          // exact for 16-bit operands; magic(0) = 2^16 excludes x == 0 (host table)
          const uint32_t m = __ldg(a.cand_magic + jg0 + c);
          ok = n * m < 0x10000u && m != 0x10000u;
        } else {
          const int32_t x = __ldg(a.cand + jg0 + c);
          const uint32_t ax = x < 0 ? 0u - (uint32_t)x : (uint32_t)x;
          ok = ax * n <= d1;  // n = ceil(2^32/d), d1 = n - 1
        }
        mask |= (uint32_t)ok << c;
      }
    }
    if (mask && a.n_terms > 1) mask = other_terms_mask(a, i, tn, jg0, mask, a.hot_term, s_opa, s_opb, s_slots, s_q);
  }
  if (mask) {
    atomicOr(&s_bm[i * RW + (jl0 >> 5)], mask << (jl0 & 31));
    atomicOr(&s_sum[i * SW + (jl0 >> 10)], 1u << ((jl0 >> 5) & 31));
    atomicAdd(&s_cnt[i], (uint32_t)__popc(mask));
  }
}

// Children of node i with a large count, emitted by the whole warp into the stash: set
// bitmap words in order, lane b writes the child of bit b (coalesced); consumed words are
// zeroed.
template <int W>
__device__ __forceinline__ void emit_node_warp(const LevelArgs& a, int i, uint64_t rank, int64_t j0, const uint32_t* rec,
                                               uint32_t* s_bm, uint32_t* s_sum, int RW, int SW, int lane) {
  const unsigned lt = (1u << lane) - 1u;
  for (int sw = 0; sw < SW; sw++) {
    uint32_t sm = s_sum[i * SW + sw];
    while (sm) {
      const int wi = sw * 32 + __ffs(sm) - 1;
      sm &= sm - 1;
      const uint32_t word = s_bm[i * RW + wi];
      if ((word >> lane) & 1u) {
        const uint64_t rk = rank + __popc(word & lt);
        if (rk < a.stash_cap) {
          const uint32_t pos = (uint32_t)(j0 + wi * 32 + lane);
          uint32_t out[W];
#pragma unroll
          for (int w = 0; w < W; w++) out[w] = rec[w] | (w == a.field_word ? pos << a.field_shift : 0u);
          store_record<W>(a.stash + rk * W, out);
        }
      }
      rank += __popc(word);
      __syncwarp();
      if (lane == 0) s_bm[i * RW + wi] = 0u;
    }
    __syncwarp();
    if (lane == 0) s_sum[i * SW + sw] = 0u;
  }
}

// ---------------------------------------------------------------- wide expand kernel
// One launch = one tree level of one group, for ranges of r > 64 candidates.  Tile =
// tile_nodes frontier nodes x one chunk of `chunk` candidates; thread t owns candidate
// positions [t*CPT, t*CPT + CPT) of the chunk.  Per tile:
//   prologue  one thread per node: path record -> ancestor values -> operands (smem)
//   hot loop  (A4) every (node, candidate) pair through the HOT filter (one IMAD + half a
//             VIMNMX3 per pair, min over the thread's candidates per node); a thread whose
//             candidates may pass for any of 4 consecutive nodes queues (node quad, thread)
//   slow path the queued pairs are evaluated exactly, one item = node x CPT candidates,
//             flattened over the block; accepted pairs set bits of a per-node candidate
//             bitmap (smem) and bump the node's count.  Queue overflow -> dense tile.
//   scan      (A5) warp scan of node counts + decoupled look-back -> CSR offsets
//   emit      (A6) lane-per-node for nodes with few children, warp-per-node (coalesced)
//             for many; records = parent record | position; consumed words are zeroed.
template <int W, int CPT, int HOT>
__global__ void __launch_bounds__(256, 4) expand_wide(const __grid_constant__ LevelArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  const SmemLayout L = expand_layout(a, W);
  uint32_t* ctl = reinterpret_cast<uint32_t*>(smem + L.ctl);
  uint32_t* s_ok = reinterpret_cast<uint32_t*>(smem + L.ok);
  uint32_t* s_rec = reinterpret_cast<uint32_t*>(smem + L.rec);
  int64_t* s_opa = reinterpret_cast<int64_t*>(smem + L.opa);
  int64_t* s_opb = reinterpret_cast<int64_t*>(smem + L.opb);
  int64_t* s_slots = L.slots >= 0 ? reinterpret_cast<int64_t*>(smem + L.slots) : nullptr;
  uint32_t* s_hot = reinterpret_cast<uint32_t*>(smem + L.hot);
  uint32_t* s_hot2 = reinterpret_cast<uint32_t*>(smem + L.hot2);
  uint32_t* s_cnt = reinterpret_cast<uint32_t*>(smem + L.cnt);
  uint32_t* s_off = reinterpret_cast<uint32_t*>(smem + L.off);
  uint32_t* s_sum = reinterpret_cast<uint32_t*>(smem + L.sum);
  uint32_t* s_bm = reinterpret_cast<uint32_t*>(smem + L.bm);
  uint32_t* s_qe = reinterpret_cast<uint32_t*>(smem + L.q);
  uint32_t* s_q = L.qtab >= 0 ? reinterpret_cast<uint32_t*>(smem + L.qtab) : nullptr;
  unsigned long long* s_w = reinterpret_cast<unsigned long long*>(smem + L.wtot);

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int B = blockDim.x, NW = B >> 5;
  const int r = a.r, NT = a.tile_nodes, RW = a.rw, SW = a.sw, chunk = a.chunk;
  const int hot_t = a.hot_term;
  constexpr uint32_t kBig = 48;  // children above which a node is emitted by the whole warp

  for (int k = tid; k < NT * RW; k += B) s_bm[k] = 0u;
  for (int k = tid; k < NT * SW; k += B) s_sum[k] = 0u;
  for (int k = tid; k < NT; k += B) s_cnt[k] = 0u;
  if (s_q)
    for (uint32_t q = tid; q <= a.qmax; q += B) s_q[q] = q ? (0xffffffffu / q + 1u) : 0u;

  // tiles by ticket, one ahead: ctl[2] = this tile, ctl[3] = the next one, whose parent
  // records are prefetched into registers during this tile's hot loop
  auto tile_nodes = [&](uint64_t t, uint64_t& n0, int64_t& c, int& cnt) {
    if (a.n_chunks == 1) {
      n0 = t * (uint64_t)NT;
      const uint64_t rem = a.n_parents - n0;
      cnt = rem < (uint64_t)NT ? (int)rem : NT;
      c = 0;
    } else {
      n0 = udiv64f(t, (uint64_t)a.n_chunks);
      c = (int64_t)umod64f(t, (uint64_t)a.n_chunks);
      cnt = 1;
    }
  };
  if (tid == 0) {
    ctl[1] = 0u;  // slow-path queue length (reset again after each tile's slow path)
    ctl[2] = atomicAdd(a.tile_counter, 1u);
    ctl[3] = atomicAdd(a.tile_counter, 1u);
  }
  __syncthreads();
  uint32_t pre[W];
  uint64_t pre_tile = ~0ull;
  for (;;) {
    const uint64_t tile = ctl[2], nxt = ctl[3];
    if (tile >= a.n_tiles) break;
    uint64_t node0;
    int64_t ch;
    int tn;
    tile_nodes(tile, node0, ch, tn);
    const int64_t j0 = ch * (int64_t)chunk;
    // ---- prologue
    for (int i = tid; i < NT; i += B) {
      if (i < tn) {
        const bool staged = a.level > 0 && i == tid && pre_tile == tile;
        if (staged) {
#pragma unroll
          for (int w = 0; w < W; w++) s_rec[i * W + w] = pre[w];
        }
        const bool ok = prologue_node<W, HOT == HOT_NONE>(a, node0 + i, i, NT, s_ok, s_rec, s_opa, s_opb, s_slots, staged);
        if (HOT == HOT_DIVX) {
          s_hot[i] = ok ? (uint32_t)s_opa[hot_t * NT + i] : kHotSentinel;
        } else if (HOT == HOT_MULX) {
          const uint32_t md = ok ? (uint32_t)s_opb[hot_t * NT + i] : (0xffffffffu / kHotSentinel + 1u);
          s_hot[i] = md;
          s_hot2[i] = md - 1u;
        }
      } else {
        s_ok[i] = 0u;
        s_hot[i] = HOT == HOT_MULX ? (0xffffffffu / kHotSentinel + 1u) : kHotSentinel;
        s_hot2[i] = (0xffffffffu / kHotSentinel);
      }
    }
    __syncthreads();
    if (tid == 0) {  // every thread has read ctl[2..3]; claim the tile after next
      ctl[2] = (uint32_t)nxt;
      ctl[3] = nxt < a.n_tiles ? atomicAdd(a.tile_counter, 1u) : (uint32_t)nxt;
    }
    if (a.level > 0 && nxt < a.n_tiles) {  // prefetch the next tile's parent records
      uint64_t n0;
      int64_t c2;
      int cnt2;
      tile_nodes(nxt, n0, c2, cnt2);
      if (tid < cnt2) {
        load_record<W>(a.parent_rec + (n0 + tid) * W, pre);
        pre_tile = nxt;
      }
    }

    // ---- hot loop (A4): superset filter, queue (node quad, thread) on a possible accept
    const bool dense = HOT == HOT_NONE;
    if (HOT != HOT_NONE) {
      //   HOT_DIVX: hm = ceil(2^32/|x|).  For 16-bit n and x, (n * hm mod 2^32) < 2^16
      //             iff x | n (exhaustively verified, tests/test_abi_cpu.py), so the
      //             per-node test is min over the candidates < 2^16: one IMAD per pair
      //             plus half a 3-input VIMNMX3.  Invalid slots and x == 0: hm = 2^16,
      //             which flags only n == 0 (the slow path rejects).
      //   HOT_MULX: hm = |x|; x * ceil(2^32/d) <= ceil(2^32/d) - 1 iff d | x, again a
      //             min over the candidates against a per-node bound.  Invalid: hm = 1.
      uint32_t hm[CPT];
#pragma unroll
      for (int c = 0; c < CPT; c++) {
        const int64_t j = j0 + tid * CPT + c;
        const bool v = j < r;
        const int32_t x = v ? __ldg(a.cand + j) : 0;
        const uint32_t ax = x < 0 ? 0u - (uint32_t)x : (uint32_t)x;
        if (HOT == HOT_DIVX) hm[c] = v ? __ldg(a.cand_magic + j) : 0x10000u;  // magic(0) = 2^16
        else hm[c] = v ? ax : 1u;
      }
      for (int g = 0; g < tn; g += 4) {
        const uint4 n4 = *reinterpret_cast<const uint4*>(s_hot + g);
        uint32_t m0 = 0xffffffffu, m1 = 0xffffffffu, m2 = 0xffffffffu, m3 = 0xffffffffu;
#pragma unroll
        for (int c = 0; c < CPT; c++) {
          m0 = min(m0, n4.x * hm[c]);
          m1 = min(m1, n4.y * hm[c]);
          m2 = min(m2, n4.z * hm[c]);
          m3 = min(m3, n4.w * hm[c]);
        }
        bool h0, h1, h2, h3;
        if (HOT == HOT_DIVX) {
          h0 = m0 < 0x10000u; h1 = m1 < 0x10000u; h2 = m2 < 0x10000u; h3 = m3 < 0x10000u;
        } else {
          const uint4 d4 = *reinterpret_cast<const uint4*>(s_hot2 + g);
          h0 = m0 <= d4.x; h1 = m1 <= d4.y; h2 = m2 <= d4.z; h3 = m3 <= d4.w;
        }
        const uint32_t hq = (uint32_t)h0 | ((uint32_t)h1 << 1) | ((uint32_t)h2 << 2) | ((uint32_t)h3 << 3);
        if (hq) {  // entry: node quad << 16 | flagged nodes << 12 | thread
          const uint32_t slot = atomicAdd(&ctl[1], 1u);
          s_qe[slot] = ((uint32_t)(g >> 2) << 16) | (hq << 12) | (uint32_t)tid;
        }
      }
      __syncthreads();
      // ---- slow path: queued (node, thread) pairs flattened over the block; one item =
      // one flagged node x the thread's CPT candidates, exact.  (qcap = one entry per
      // node quad and thread, so the queue cannot overflow.)
      const uint32_t items = ctl[1] * 4u;
      for (uint32_t k = tid; k < items; k += B) {
        const uint32_t e = s_qe[k >> 2];
        if (!((e >> (12 + (k & 3u))) & 1u)) continue;
        const int i = (int)((e >> 16) * 4u + (k & 3u));
        const int jl0 = (int)((e & 0xfffu) * CPT);
        record_mask<CPT, HOT>(a, i, NT, jl0, j0, s_ok, s_hot, s_hot2, s_opa, s_opb, s_slots, s_q, s_bm, s_sum,
                              s_cnt, RW, SW);
      }
    }
    if (dense) {
      // every (node, candidate) pair of the tile exactly; thread-owned candidates
      const int jl0 = tid * CPT;
      for (int i = 0; i < tn; i++)
        record_mask<CPT, HOT>(a, i, NT, jl0, j0, s_ok, s_hot, s_hot2, s_opa, s_opb, s_slots, s_q, s_bm, s_sum,
                              s_cnt, RW, SW);
    }
    __syncthreads();

    // ---- scan (A5, tile part): node counts -> tile-local offsets; the tile's children
    // go to a stash segment claimed with one atomic (no wait on other tiles); the
    // device-wide scan of tile totals and the copy to final positions follow in
    // scan_kernel + wide_emit_kernel.
    if (warp == 0) {
      uint32_t run = 0;
      for (int i0 = 0; i0 < tn; i0 += 32) {
        const int i = i0 + lane;
        const uint32_t v = i < tn ? s_cnt[i] : 0u;
        uint32_t incl = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(FULL, incl, o);
          if (lane >= o) incl += y;
        }
        if (i < tn) s_off[i] = run + incl - v;
        run += __shfl_sync(FULL, incl, 31);
      }
      if (lane == 0) {
        ctl[1] = 0u;  // queue consumed (barrier after the slow path); next tile's hot loop is 2 barriers away
        const unsigned long long seg = run ? atomicAdd(a.stash_top, (unsigned long long)run) : 0ull;
        if (run && seg + run > a.stash_cap) atomicOr(a.overflow_flag, 1u);
        a.tile_total[tile] = run;
        a.tile_seg[tile] = seg;
        s_w[33] = seg;
      }
    }
    __syncthreads();
    const uint64_t seg = s_w[33];

    // ---- emit (A6, into the stash segment in final order); CSR gets tile-local offsets
    if (ch == 0)
      for (int i = tid; i < tn; i += B) a.csr[node0 + i] = s_off[i];
    for (int i0 = warp * 32; i0 < tn; i0 += NW * 32) {
      const int i = i0 + lane;
      const uint32_t cnt = i < tn ? s_cnt[i] : 0u;
      if (cnt && cnt <= kBig) {
        // lane per node: its set words in order, its bits in order
        uint64_t rank = seg + s_off[i];
        uint32_t rec[W];
#pragma unroll
        for (int w = 0; w < W; w++) rec[w] = s_rec[i * W + w];
        for (int sw = 0; sw < SW; sw++) {
          uint32_t sm = s_sum[i * SW + sw];
          if (!sm) continue;
          s_sum[i * SW + sw] = 0u;
          while (sm) {
            const int wi = sw * 32 + __ffs(sm) - 1;
            sm &= sm - 1;
            uint32_t word = s_bm[i * RW + wi];
            s_bm[i * RW + wi] = 0u;
            while (word) {
              const int b = __ffs(word) - 1;
              word &= word - 1;
              if (rank < a.stash_cap) {
                const uint32_t pos = (uint32_t)(j0 + wi * 32 + b);
                uint32_t out[W];
#pragma unroll
                for (int w = 0; w < W; w++) out[w] = rec[w] | (w == a.field_word ? pos << a.field_shift : 0u);
                store_record<W>(a.stash + rank * W, out);
              }
              rank++;
            }
          }
        }
      }
      unsigned big = __ballot_sync(FULL, cnt > kBig);
      while (big) {
        const int src = __ffs(big) - 1;
        big &= big - 1;
        const int ib = i0 + src;
        uint32_t rec[W];
#pragma unroll
        for (int w = 0; w < W; w++) rec[w] = s_rec[ib * W + w];
        emit_node_warp<W>(a, ib, seg + s_off[ib], j0, rec, s_bm, s_sum, RW, SW, lane);
      }
      if (i < tn) s_cnt[i] = 0u;
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- warp-tile expand kernel
// One launch = one tree level of one group, for 64 < r <= kMaxSeg * 32 * CPT.  Every warp
// works alone on tiles of kWT = 32 consecutive frontier nodes x all r candidates (no block
// barrier after the candidate table is staged), so the scheduler always has independent
// warps to issue from.  Candidate position j = seg * 32 * CPT + b * CPT + c: lane b owns
// CPT consecutive candidates of every segment.  Per tile:
//   prologue  lane i: node i's path record -> ancestor values -> operands (warp region)
//   hot loop  (A4) per segment, per node quad: one IMAD + half a VIMNMX3 per pair (the
//             expand_wide filter); the per-node ballot of "some candidate of lane b may
//             pass" is the node's item word for the segment (item = node x seg x lane)
//   items     the tile's items in canonical order (node, seg, lane) = candidate order;
//             rounds of 32 items, one per lane: exact accept mask of the item's CPT
//             candidates (hot conjunct from the table, other conjuncts on survivors)
//   scan      (A5) warp scan of node counts -> tile-local CSR; one atomicAdd claims the
//             tile's stash segment (no wait on other tiles)
//   emit      (A6) warp scan of item counts -> each lane writes its item's children
//             (records = parent record | position) in final order into the segment
// scan_kernel + level_emit_kernel then place the segments (as for the other kernels).

// position of the (n+1)-th set bit of w (n < popc(w))
__device__ __forceinline__ int nth_set_bit(uint32_t w, int n) {
  int pos = 0;
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) {
    const int c = __popc(w & ((1u << s) - 1u));
    if (n >= c) { n -= c; w >>= s; pos += s; }
  }
  return pos;
}

template <int CPT, int HOT>
__device__ __forceinline__ uint32_t wtile_item_mask(const LevelArgs& a, int i, int sg, int b, const uint32_t* s_tab,
                                                    const uint32_t* s_ok, const uint32_t* s_hot,
                                                    const uint32_t* s_hot2, const int64_t* s_opa,
                                                    const int64_t* s_opb, const int64_t* s_slots,
                                                    const uint32_t* s_q) {
  constexpr int SEG = 32 * CPT;
  const int64_t jl = (int64_t)sg * SEG + (int64_t)b * CPT;
  const int64_t left = (int64_t)a.r - jl;
  const uint32_t valid = left >= CPT ? (CPT == 32 ? 0xffffffffu : ((1u << CPT) - 1u))
                                     : (left > 0 ? ((1u << left) - 1u) : 0u);
  uint32_t mask = 0;
  if (HOT == HOT_NONE) {
    if (a.n_terms == 0) return valid;  // unconstrained level (node gates already applied)
#pragma unroll 4
    for (int c = 0; c < CPT; c++)
      if (((valid >> c) & 1u) &&
          node_accepts(a, i, kWT, __ldg(a.cand + jl + c), __ldg(a.cand_magic + jl + c), s_ok, s_opa, s_opb, s_slots,
                       s_q))
        mask |= 1u << c;
    return mask;
  }
  const uint32_t n = s_hot[i], d1 = s_hot2[i];
  const uint32_t* tp = s_tab + sg * SEG + b;
#pragma unroll
  for (int c = 0; c < CPT; c++) {
    const uint32_t t = tp[c * 32];
    bool ok;
    if (HOT == HOT_DIVX) ok = n * t < 0x10000u && t != 0x10000u;  // x | n, exact for 16-bit operands
    else ok = t * n <= d1;                                          // d | x, n = ceil(2^32/d)
    mask |= (uint32_t)ok << c;
  }
  mask &= valid;
  if (mask && a.n_terms > 1) mask = other_terms_mask(a, i, kWT, jl, mask, a.hot_term, s_opa, s_opb, s_slots, s_q);
  return mask;
}

// Item k of the tile -> (node, segment, lane b).  ie: this lane's exclusive item prefix
// (lane = node); nodes without items share the next node's prefix, so the largest node
// whose prefix is <= k owns item k.
template <int HOT>
__device__ __forceinline__ void wtile_decode_item(uint32_t k, uint32_t ie, const uint32_t* s_items, int nseg,
                                                  uint32_t vword_last, int& node, int& sg, int& b) {
  int nd = 0;
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) {
    const uint32_t e = __shfl_sync(FULL, ie, (nd + s) & 31);
    if (nd + s < 32 && e <= k) nd += s;
  }
  int rr = (int)(k - __shfl_sync(FULL, ie, nd));
  node = nd;
  sg = 0;
  b = 0;
  for (int q = 0; q < nseg; q++) {
    const uint32_t w = HOT == HOT_NONE ? (q == nseg - 1 ? vword_last : 0xffffffffu) : s_items[q * kWT + nd];
    const int p = __popc(w);
    if (rr < p) {
      sg = q;
      b = nth_set_bit(w, rr);
      break;
    }
    rr -= p;
  }
}

template <int W, int CPT, int HOT>
__global__ void __launch_bounds__(256, 3) expand_wtile(const __grid_constant__ LevelArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  constexpr int SEG = 32 * CPT;
  const WarpLayout L = wtile_layout(a, W);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int nseg = a.nseg, r = a.r, hot_t = a.hot_term;
  const int TN = a.tile_nodes;  // nodes per warp tile (power of two <= kWT; small levels use fewer)
  uint32_t* s_tab = L.tab >= 0 ? reinterpret_cast<uint32_t*>(smem + L.tab) : nullptr;
  uint32_t* s_q = L.qtab >= 0 ? reinterpret_cast<uint32_t*>(smem + L.qtab) : nullptr;
  if (HOT != HOT_NONE) {
    // hot operand per candidate slot, transposed [seg][c][lane]; padding: magic(0) = 2^16
    // (DIVX) / |x| = 1 (MULX), rejected by the exact test's validity mask
    const uint32_t* src = HOT == HOT_DIVX ? a.cand_magic : a.cand_abs;
    const uint32_t pad = HOT == HOT_DIVX ? 0x10000u : 1u;
    for (int j = threadIdx.x; j < nseg * SEG; j += blockDim.x) {
      const int sg = j / SEG, rem = j - sg * SEG, b = rem / CPT, c = rem - b * CPT;
      s_tab[sg * SEG + c * 32 + b] = j < r ? __ldg(src + j) : pad;
    }
  }
  if (s_q)
    for (uint32_t q = threadIdx.x; q <= a.qmax; q += blockDim.x) s_q[q] = q ? (0xffffffffu / q + 1u) : 0u;
  __syncthreads();  // the only block barrier: everything below is per warp

  unsigned char* wb = smem + L.warp0 + warp * L.wstride;
  uint32_t* s_rec = reinterpret_cast<uint32_t*>(wb + L.rec);
  uint32_t* s_ok = reinterpret_cast<uint32_t*>(wb + L.ok);
  uint32_t* s_hot = reinterpret_cast<uint32_t*>(wb + L.hot);
  uint32_t* s_hot2 = reinterpret_cast<uint32_t*>(wb + L.hot2);
  uint32_t* s_cnt = reinterpret_cast<uint32_t*>(wb + L.cnt);
  uint32_t* s_items = reinterpret_cast<uint32_t*>(wb + L.items);
  uint32_t* s_imask = reinterpret_cast<uint32_t*>(wb + L.imask);
  uint16_t* s_icode = reinterpret_cast<uint16_t*>(wb + L.icode);
  int64_t* s_opa = reinterpret_cast<int64_t*>(wb + L.opa);
  int64_t* s_opb = reinterpret_cast<int64_t*>(wb + L.opb);
  int64_t* s_slots = L.slots >= 0 ? reinterpret_cast<int64_t*>(wb + L.slots) : nullptr;
  s_cnt[lane] = 0u;
  // valid-lane word of the last segment (dense levels: every valid pair is an item)
  const int64_t last_left = (int64_t)r - (int64_t)(nseg - 1) * SEG;  // candidates in the last segment
  const int last_lanes = (int)((last_left + CPT - 1) / CPT);
  const uint32_t vword_last = last_lanes >= 32 ? 0xffffffffu : ((1u << last_lanes) - 1u);

  uint32_t cur = 0, nxt = 0;
  if (lane == 0) {
    cur = atomicAdd(a.tile_counter, 1u);
    nxt = atomicAdd(a.tile_counter, 1u);
  }
  cur = __shfl_sync(FULL, cur, 0);
  nxt = __shfl_sync(FULL, nxt, 0);
  uint32_t pre[W];
  uint64_t pre_tile = ~0ull;
  uint64_t pairs = 0;  // hot-loop pairs tested (ATF_FLAG_TIMING statistics)
  while ((uint64_t)cur < a.n_tiles) {
    const uint64_t node0 = (uint64_t)cur * TN;
    const uint64_t remn = a.n_parents - node0;
    const int tn = remn < (uint64_t)TN ? (int)remn : TN;
    // ---- prologue: lane = node
    bool ok = false;
    if (lane < tn) {
      const bool staged = a.level > 0 && pre_tile == cur;
      if (staged) {
#pragma unroll
        for (int w = 0; w < W; w++) s_rec[lane * W + w] = pre[w];
      }
      ok = prologue_node<W, HOT == HOT_NONE>(a, node0 + lane, lane, kWT, s_ok, s_rec, s_opa, s_opb, s_slots, staged);
    } else {
      s_ok[lane] = 0u;
    }
    if (HOT == HOT_DIVX) {
      s_hot[lane] = ok ? (uint32_t)s_opa[hot_t * kWT + lane] : kHotSentinel;
    } else if (HOT == HOT_MULX) {
      const uint32_t md = ok ? (uint32_t)s_opb[hot_t * kWT + lane] : (0xffffffffu / kHotSentinel + 1u);
      s_hot[lane] = md;
      s_hot2[lane] = md - 1u;
    }
    // segment bounds of the hot filter (A4): x | n (n != 0) needs |x| <= n, d | x (x != 0)
    // needs |x| >= d, so a node quad whose largest n (smallest d) lies outside a segment's
    // [seg_lo, seg_hi] has no item there.  Lane 4q holds quad q's bound; rejected nodes
    // bound nothing, n == 0 (divisible by every x) bounds everything.
    uint32_t qb = 0;
    if (HOT == HOT_DIVX) {
      qb = ok ? (s_hot[lane] ? s_hot[lane] : 0xffffffffu) : 0u;
      qb = max(qb, __shfl_xor_sync(FULL, qb, 1));
      qb = max(qb, __shfl_xor_sync(FULL, qb, 2));
    } else if (HOT == HOT_MULX) {
      qb = ok ? (uint32_t)s_opa[hot_t * kWT + lane] : 0xffffffffu;
      qb = min(qb, __shfl_xor_sync(FULL, qb, 1));
      qb = min(qb, __shfl_xor_sync(FULL, qb, 2));
    }
    // claim the tile after next; prefetch the next tile's parent records
    uint32_t nn = nxt;
    if (lane == 0 && (uint64_t)nxt < a.n_tiles) nn = atomicAdd(a.tile_counter, 1u);
    nn = __shfl_sync(FULL, nn, 0);
    if (a.level > 0 && (uint64_t)nxt < a.n_tiles) {
      const uint64_t n1 = (uint64_t)nxt * TN + lane;
      if (lane < TN && n1 < a.n_parents) {
        load_record<W>(a.parent_rec + n1 * W, pre);
        pre_tile = nxt;
      }
    }
    __syncwarp();

    // ---- hot loop (A4): item words = per-node ballots of the superset filter
    const int nq = (tn + 3) >> 2;
    if (HOT != HOT_NONE) {
      const bool seg_on = a.seg_on != 0;  // segment bounds in force (not the headline flags)
      pairs += (uint64_t)tn * (uint64_t)r;  // less the pairs of skipped quad segments below
      for (int sg = 0; sg < nseg; sg++) {
        uint32_t hm[CPT];
        const uint32_t* tp = s_tab + sg * SEG + lane;
#pragma unroll
        for (int c = 0; c < CPT; c++) hm[c] = tp[c * 32];
        uint32_t sb = 0;
        if (seg_on) {
          sb = HOT == HOT_DIVX ? a.seg_lo[0] : a.seg_hi[0];  // no dynamic param indexing
#pragma unroll
          for (int i = 1; i < kMaxSeg; i++)
            if (sg == i) sb = HOT == HOT_DIVX ? a.seg_lo[i] : a.seg_hi[i];
        }
        for (int q = 0; q < nq; q++) {
          if (seg_on) {
            const uint32_t qv = __shfl_sync(FULL, qb, 4 * q);
            if (HOT == HOT_DIVX ? qv < sb : qv > sb) {
              if (lane == 0) *reinterpret_cast<uint4*>(s_items + sg * kWT + 4 * q) = make_uint4(0u, 0u, 0u, 0u);
              pairs -= (uint64_t)min(4, tn - 4 * q) * (uint64_t)min(SEG, r - sg * SEG);
              continue;
            }
          }
          const uint4 n4 = *reinterpret_cast<const uint4*>(s_hot + 4 * q);
          uint32_t m0 = 0xffffffffu, m1 = 0xffffffffu, m2 = 0xffffffffu, m3 = 0xffffffffu;
#pragma unroll
          for (int c = 0; c < CPT; c++) {
            m0 = min(m0, n4.x * hm[c]);
            m1 = min(m1, n4.y * hm[c]);
            m2 = min(m2, n4.z * hm[c]);
            m3 = min(m3, n4.w * hm[c]);
          }
          bool h0, h1, h2, h3;
          if (HOT == HOT_DIVX) {
            h0 = m0 < 0x10000u; h1 = m1 < 0x10000u; h2 = m2 < 0x10000u; h3 = m3 < 0x10000u;
          } else {
            const uint4 d4 = *reinterpret_cast<const uint4*>(s_hot2 + 4 * q);
            h0 = m0 <= d4.x; h1 = m1 <= d4.y; h2 = m2 <= d4.z; h3 = m3 <= d4.w;
          }
          const uint32_t b0 = __ballot_sync(FULL, h0), b1 = __ballot_sync(FULL, h1);
          const uint32_t b2 = __ballot_sync(FULL, h2), b3 = __ballot_sync(FULL, h3);
          if (lane == 0) *reinterpret_cast<uint4*>(s_items + sg * kWT + 4 * q) = make_uint4(b0, b1, b2, b3);
        }
      }
      __syncwarp();
    }

    // ---- items: per-node item counts (lane = node) -> exclusive item prefix
    uint32_t ic = 0;
    if (lane < tn && s_ok[lane]) {
      if (HOT == HOT_NONE) {
        ic = (uint32_t)(nseg - 1) * 32u + (uint32_t)__popc(vword_last);
      } else {
        for (int sg = 0; sg < nseg; sg++) ic += (uint32_t)__popc(s_items[sg * kWT + lane]);
      }
    }
    uint32_t ie = ic;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL, ie, o);
      if (lane >= o) ie += y;
    }
    const uint32_t T = __shfl_sync(FULL, ie, 31);
    ie -= ic;
    // pass 1: exact masks -> node counts; the first kItemCap items keep (mask, item code =
    // node | seg << 5 | lane << 8) in the warp's shared memory for the emit pass
    for (uint32_t R = 0; R < T; R += 32) {
      const uint32_t k = R + lane;
      int node, sg, b;
      wtile_decode_item<HOT>(k < T ? k : T - 1, ie, s_items, nseg, vword_last, node, sg, b);
      uint32_t m = 0;
      if (k < T)
        m = wtile_item_mask<CPT, HOT>(a, node, sg, b, s_tab, s_ok, s_hot, s_hot2, s_opa, s_opb, s_slots, s_q);
      if (k < (uint32_t)kItemCap) {
        s_imask[k] = m;
        s_icode[k] = (uint16_t)((uint32_t)node | ((uint32_t)sg << 5) | ((uint32_t)b << 8));
      }
      if (m) atomicAdd(&s_cnt[node], (uint32_t)__popc(m));
    }
    __syncwarp();
    // ---- scan (A5, tile part): node counts -> tile-local CSR offsets, stash segment
    const uint32_t cn = lane < tn ? s_cnt[lane] : 0u;
    uint32_t co = cn;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL, co, o);
      if (lane >= o) co += y;
    }
    const uint32_t total = __shfl_sync(FULL, co, 31);
    s_cnt[lane] = 0u;  // for the next tile (read above by this lane only)
    unsigned long long sgb = 0;
    uint32_t* dst = a.stash;
    uint64_t cap = a.stash_cap;
    if (a.direct) {
      // tiny level (a handful of tiles, all resident): the tile's final base by decoupled
      // look-back; children and CSR entries go straight to their final place (no scan /
      // copy launches)
      sgb = lookback(a.status, cur, total, lane);
      dst = a.child_rec;
      cap = a.child_cap;
      if (lane < tn) a.csr[node0 + lane] = sgb + co - cn;
      if (lane == 0) {
        if (sgb + total > cap) atomicOr(a.overflow_flag, 1u);
        if ((uint64_t)cur == a.n_tiles - 1) {
          *a.total_out = sgb + total;
          a.csr[a.n_parents] = sgb + total;
        }
      }
    } else {
      if (lane < tn) a.csr[node0 + lane] = co - cn;
      if (lane == 0) {
        sgb = total ? atomicAdd(a.stash_top, (unsigned long long)total) : 0ull;
        if (total && sgb + total > a.stash_cap) atomicOr(a.overflow_flag, 1u);
        a.tile_total[cur] = total;
        a.tile_seg[cur] = sgb;
      }
      sgb = __shfl_sync(FULL, sgb, 0);
    }
    // ---- emit (A6): items in order; lane writes its item's children at their final rank
    uint64_t carry = sgb;
    for (uint32_t R = 0; R < T; R += 32) {
      const uint32_t k = R + lane;
      int node, sg, b;
      uint32_t m;
      if (R < (uint32_t)kItemCap) {
        const uint32_t code = s_icode[k];
        m = k < T ? s_imask[k] : 0u;
        node = (int)(code & 31u);
        sg = (int)((code >> 5) & 7u);
        b = (int)(code >> 8);
      } else {
        wtile_decode_item<HOT>(k < T ? k : T - 1, ie, s_items, nseg, vword_last, node, sg, b);
        m = k < T ? wtile_item_mask<CPT, HOT>(a, node, sg, b, s_tab, s_ok, s_hot, s_hot2, s_opa, s_opb, s_slots, s_q)
                  : 0u;
      }
      const uint32_t pc = (uint32_t)__popc(m);
      uint32_t incl = pc;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
      }
      uint64_t rank = carry + (incl - pc);
      carry += __shfl_sync(FULL, incl, 31);
      if (m) {
        uint32_t rec[W];
#pragma unroll
        for (int w = 0; w < W; w++) rec[w] = s_rec[node * W + w];
        const uint32_t pos0 = (uint32_t)(sg * SEG + b * CPT);
        while (m) {
          const int c = __ffs(m) - 1;
          m &= m - 1;
          if (rank < cap) {
            uint32_t out[W];
#pragma unroll
            for (int w = 0; w < W; w++) out[w] = rec[w] | (w == a.field_word ? (pos0 + c) << a.field_shift : 0u);
            store_record<W>(dst + rank * W, out);
          }
          rank++;
        }
      }
    }
    __syncwarp();
    cur = nxt;
    nxt = nn;
  }
  if (a.pairs_out && lane == 0 && pairs) atomicAdd(a.pairs_out, (unsigned long long)pairs);
}

template <typename K>
static int launch_persistent(K k, const LevelArgs& a, int block, void* stream) {
  const int smem = a.smem_bytes;
  const int per_sm = cached_occupancy((const void*)k, block, smem);
  if (per_sm < 0) return -per_sm;
  if (per_sm < 1) return (int)cudaErrorInvalidConfiguration;
  uint64_t grid = (uint64_t)cached_sm_count() * per_sm;  // persistent: one wave, tiles by ticket
  if (grid > a.n_tiles) grid = a.n_tiles;
  if (grid < 1) grid = 1;
  k<<<(unsigned)grid, block, smem, (cudaStream_t)stream>>>(a);
  return (int)cudaGetLastError();
}

template <int W, int CPT>
static int launch_wide_wc(const LevelArgs& a, void* stream) {
  switch (a.hot) {
    case HOT_NONE: return launch_persistent(expand_wide<W, CPT, HOT_NONE>, a, a.block, stream);
    case HOT_DIVX: return launch_persistent(expand_wide<W, CPT, HOT_DIVX>, a, a.block, stream);
    case HOT_MULX: return launch_persistent(expand_wide<W, CPT, HOT_MULX>, a, a.block, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

// ---------------------------------------------------------------- narrow fast kernel
// r <= 32 candidates and a level whose conjuncts are all 16/32-bit atoms over ancestor
// values, constants or products of two ancestors (host: nf_ok; every C1-C3 narrow level).
// Warp-autonomous tiles of 32 x kNfNPL frontier nodes (lane l: nodes l, l+32, ...); per
// node the operands come straight from the parent record (field -> range value, and the
// range's divisor magic where a quotient or a d | x test needs one: no division, no
// per-node slot array), each conjunct is a bit-parallel mask over the r candidates
// (candidate values / magics in shared memory), children are written by their node's
// lane in candidate order into the tile's stash segment.  No block barrier after staging.
template <int W>
__device__ __forceinline__ uint32_t nf_field(const LevelArgs& a, const uint32_t* rec, int s) {
  uint32_t word = rec[0];
#pragma unroll
  for (int w = 1; w < W; w++)
    if (a.pv_word[s] == w) word = rec[w];
  const uint32_t bits = (uint32_t)a.pv_bits[s];
  return bits ? (word >> a.pv_shift[s]) & ((1u << bits) - 1u) : 0u;
}
// signed value of operand o
template <int W>
__device__ __forceinline__ int64_t nf_sval(const LevelArgs& a, const NfOp& o, const uint32_t* rec) {
  if (o.kind == NF_CONST) return o.c;
  const int64_t v1 = __ldg(a.pv_range[o.s1] + nf_field<W>(a, rec, o.s1));
  if (o.kind == NF_PV) return v1;
  return v1 * (int64_t)__ldg(a.pv_range[o.s2] + nf_field<W>(a, rec, o.s2));
}
// |value| of operand o and its divisor magic ceil(2^32/|v|) mod 2^32 (0 for |v| <= 1)
template <int W>
__device__ __forceinline__ uint32_t nf_abs(const LevelArgs& a, const NfOp& o, const uint32_t* rec, uint32_t* mag) {
  if (o.kind == NF_CONST) {
    if (mag) *mag = o.cm;
    return o.c < 0 ? 0u - (uint32_t)o.c : (uint32_t)o.c;
  }
  if (o.kind == NF_PV) {
    const uint32_t pos = nf_field<W>(a, rec, o.s1);
    const int32_t v = __ldg(a.pv_range[o.s1] + pos);
    const uint32_t av = v < 0 ? 0u - (uint32_t)v : (uint32_t)v;
    if (mag) *mag = av == 0 ? 0u : __ldg(a.pv_magic[o.s1] + pos);
    return av;
  }
  const int64_t p = nf_sval<W>(a, o, rec);
  const uint32_t av = (uint32_t)(p < 0 ? -p : p);
  if (mag) *mag = av > 1 ? 0xffffffffu / av + 1u : 0u;
  return av;
}

template <int W, typename M>
__device__ __forceinline__ M nf_node_mask(const LevelArgs& a, const uint32_t* rec, int r, M m, M nz, const int32_t* s_cx, const uint32_t* s_cm,
                                                 const uint32_t* s_ca) {
  for (int t = 0; t < a.n_terms && m; t++) {
    const Term& T = a.terms[t];
    const NfOp& oa = a.nf_op[t][0];
    const NfOp& ob = a.nf_op[t][1];
    M mm = 0;
    switch (T.kind) {
      case T_DIVX:
      case T_DIVPROD: {  // x | n; DIVPROD: gate a != 0 && a | b, n = b / a (magic quotient)
        uint32_t n;
        if (T.kind == T_DIVX) {
          n = nf_abs<W>(a, oa, rec, nullptr);
        } else {
          uint32_t ma;
          const uint32_t av = nf_abs<W>(a, oa, rec, &ma), bv = nf_abs<W>(a, ob, rec, nullptr);
          if (av == 0) return 0;
          n = av == 1 ? bv : __umulhi(bv, ma);
          if (n * av != bv) return 0;
        }
#pragma unroll 4
        for (int c = 0; c < r; c++) mm |= (M)(n * s_cm[c] < 0x10000u) << c;
        mm &= nz;  // x == 0 rejects (poison)
        break;
      }
      case T_MULX: {  // d | x, d != 0
        uint32_t md;
        const uint32_t d = nf_abs<W>(a, oa, rec, &md);
        if (d == 0) return 0;
        const uint32_t md1 = md - 1u;
#pragma unroll 4
        for (int c = 0; c < r; c++) mm |= (M)(s_ca[c] * md <= md1) << c;
        break;
      }
      case T_QDIV: {  // (num / x) | nb; x == 0 or quotient 0 rejects
        const uint32_t num = nf_abs<W>(a, oa, rec, nullptr), nb = nf_abs<W>(a, ob, rec, nullptr);
        M rest = m;
        while (rest) {
          const int c = (sizeof(M) == 8 ? __ffsll((long long)rest) : __ffs((int)rest)) - 1;
          rest &= rest - 1;
          const uint32_t ax = s_ca[c];
          if (ax == 0) continue;
          const uint32_t q = ax == 1 ? num : __umulhi(num, s_cm[c]);
          if (q != 0 && divisible16(nb, q)) mm |= (M)1 << c;
        }
        break;
      }
      default: {  // T_CMP, 32-bit: (A * x) rel B
        const int32_t A = (int32_t)nf_sval<W>(a, oa, rec), Bv = (int32_t)nf_sval<W>(a, ob, rec);
#pragma unroll 4
        for (int c = 0; c < r; c++) mm |= (M)rel_holds32(T.rel, A * s_cx[c], Bv) << c;
        break;
      }
    }
    m &= mm;
  }
  return m;
}

// Pass 1 (A4): accept masks of every frontier node (mask_bytes = 1/2/4/8 per node) and the
// child count of every warp tile (tile_total).  Tiles are static: warp w of the grid takes
// tiles w, w + nwarps, ...
template <int W, typename M>
__global__ void __launch_bounds__(256, 4) expand_nfast(const __grid_constant__ LevelArgs a) {
  __shared__ int32_t s_cx[64];
  __shared__ uint32_t s_cm[64], s_ca[64];
  const int lane = threadIdx.x & 31;
  const int r = a.r;
  if (threadIdx.x < 64) {
    const bool v = threadIdx.x < r;
    s_cx[threadIdx.x] = v ? __ldg(a.cand + threadIdx.x) : 0;
    s_cm[threadIdx.x] = v ? __ldg(a.cand_magic + threadIdx.x) : 0x10000u;
    s_ca[threadIdx.x] = v ? __ldg(a.cand_abs + threadIdx.x) : 0u;
  }
  __syncthreads();
  const M full = r >= (int)(8 * sizeof(M)) ? ~(M)0 : (((M)1 << r) - 1);
  M nz = 0;
  for (int c = 0; c < r; c++) nz |= (M)(s_cx[c] != 0) << c;
  constexpr int TN = 32 * kNfNPL;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t t = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; t < a.n_tiles; t += nw) {
    const uint64_t node0 = t * TN;
    uint32_t rec[kNfNPL][W];
#pragma unroll
    for (int q = 0; q < kNfNPL; q++) {
      const uint64_t nd = node0 + (uint64_t)q * 32 + lane;
      if (nd < a.n_parents) {
        if (a.level == 0) {
#pragma unroll
          for (int w = 0; w < W; w++) rec[q][w] = 0u;
        } else {
          load_record<W>(a.parent_rec + nd * W, rec[q]);
        }
      }
    }
    uint32_t cnt = 0;
#pragma unroll
    for (int q = 0; q < kNfNPL; q++) {
      const uint64_t nd = node0 + (uint64_t)q * 32 + lane;
      if (nd < a.n_parents) {
        const M m = nf_node_mask<W, M>(a, rec[q], r, full, nz, s_cx, s_cm, s_ca);
        cnt += (uint32_t)__popcll((unsigned long long)m);
        if (a.mask_bytes == 1) reinterpret_cast<uint8_t*>(a.masks)[nd] = (uint8_t)m;
        else if (a.mask_bytes == 2) reinterpret_cast<uint16_t*>(a.masks)[nd] = (uint16_t)m;
        else if (a.mask_bytes == 4) reinterpret_cast<uint32_t*>(a.masks)[nd] = (uint32_t)m;
        else reinterpret_cast<unsigned long long*>(a.masks)[nd] = (unsigned long long)m;
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(FULL, cnt, o);
    if (lane == 0) a.tile_total[t] = cnt;
  }
}

// Pass 2 (A6, after scan_kernel turned tile_total into tile_base): children written at
// their final index, CSR entries final; no stash.  A warp tile's children (<= 4 KB) are
// assembled in the warp's shared-memory buffer in order and written out as coalesced
// vectors; larger tiles write each child directly.
constexpr int kNfEmitBufBytes = 4096;  // per warp

template <int W>
__global__ void __launch_bounds__(256) nfast_emit(const __grid_constant__ LevelArgs a) {
  extern __shared__ __align__(16) unsigned char nf_smem[];
  using V = typename std::conditional<W == 1, uint32_t, typename std::conditional<W == 2, uint2, uint4>::type>::type;
  constexpr int VPR = W == 8 ? 2 : 1;                        // vectors per record
  constexpr int CAP = kNfEmitBufBytes / (4 * W);             // records per warp buffer
  const int lane = threadIdx.x & 31;
  uint32_t* buf = reinterpret_cast<uint32_t*>(nf_smem + (threadIdx.x >> 5) * kNfEmitBufBytes);
  constexpr int TN = 32 * kNfNPL;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t total = a.tile_base[a.n_tiles];
  if (gw == 0 && lane == 0) {
    if (total > a.child_cap) atomicOr(a.overflow_flag, 1u);
    *a.total_out = total;
    a.csr[a.n_parents] = total;
  }
  if (total > a.child_cap) return;
  for (uint64_t t = gw; t < a.n_tiles; t += nw) {
    const uint64_t node0 = t * TN;
    unsigned long long mask[kNfNPL];
    uint32_t rec[kNfNPL][W];
#pragma unroll
    for (int q = 0; q < kNfNPL; q++) {
      const uint64_t nd = node0 + (uint64_t)q * 32 + lane;
      mask[q] = 0;
      if (nd < a.n_parents) {
        if (a.mask_bytes == 1) mask[q] = reinterpret_cast<const uint8_t*>(a.masks)[nd];
        else if (a.mask_bytes == 2) mask[q] = reinterpret_cast<const uint16_t*>(a.masks)[nd];
        else if (a.mask_bytes == 4) mask[q] = reinterpret_cast<const uint32_t*>(a.masks)[nd];
        else mask[q] = reinterpret_cast<const unsigned long long*>(a.masks)[nd];
      }
    }
#pragma unroll
    for (int q = 0; q < kNfNPL; q++) {
      const uint64_t nd = node0 + (uint64_t)q * 32 + lane;
      if (mask[q]) {
        if (a.level == 0) {
#pragma unroll
          for (int w = 0; w < W; w++) rec[q][w] = 0u;
        } else {
          load_record<W>(a.parent_rec + nd * W, rec[q]);
        }
      }
    }
    const uint64_t base = a.tile_base[t];
    const uint32_t tt = (uint32_t)(a.tile_base[t + 1] - base);  // the tile's children
    const bool staged = tt <= (uint32_t)CAP;
    const bool coop = tt >= 32u * (uint32_t)TN;
    uint32_t run = 0;
#pragma unroll
    for (int q = 0; q < kNfNPL; q++) {
      const uint64_t nd = node0 + (uint64_t)q * 32 + lane;
      const uint32_t c = (uint32_t)__popcll(mask[q]);
      uint32_t incl = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
      }
      uint32_t rank = run + (incl - c);  // tile-local
      run += __shfl_sync(FULL, incl, 31);
      if (nd < a.n_parents) a.csr[nd] = base + rank;
      if (coop) {
        // a dense tile (>= 32 children per parent on average, C3-IS4's unconstrained KWG level):
        // the warp writes each node's children together -- lane l takes candidate bits l and
        // l + 32 -- so the stores are coalesced instead of every lane walking its own node's mask
        // (32 scattered streams): C3-IS4 1.54 -> 1.50 ms; sparser tiles keep the per-lane walk
        for (int src = 0; src < 32; src++) {
          const unsigned long long ms = __shfl_sync(FULL, mask[q], src);
          if (!ms) continue;  // warp-uniform
          const uint32_t r0 = __shfl_sync(FULL, rank, src);
          uint32_t rr[W];
#pragma unroll
          for (int w = 0; w < W; w++) rr[w] = __shfl_sync(FULL, rec[q][w], src);
#pragma unroll
          for (int h = 0; h < 2; h++) {
            if (h == 1 && a.r <= 32) break;  // (warp-uniform) no candidate bits above 31
            const int pos = lane + 32 * h;
            if ((ms >> pos) & 1ull) {
              const uint32_t k = (uint32_t)__popcll(ms & ((1ull << pos) - 1ull));
              uint32_t out[W];
#pragma unroll
              for (int w = 0; w < W; w++) out[w] = rr[w] | (w == a.field_word ? (uint32_t)pos << a.field_shift : 0u);
              store_record<W>(a.child_rec + (base + r0 + k) * W, out);
            }
          }
        }
        continue;
      }
      unsigned long long m = mask[q];
      while (m) {
        const int cc = __ffsll((long long)m) - 1;
        m &= m - 1;
        uint32_t out[W];
#pragma unroll
        for (int w = 0; w < W; w++) out[w] = rec[q][w] | (w == a.field_word ? (uint32_t)cc << a.field_shift : 0u);
        if (staged) {
#pragma unroll
          for (int w = 0; w < W; w++) buf[rank * W + w] = out[w];
        } else {
          store_record<W>(a.child_rec + (base + rank) * W, out);
        }
        rank++;
      }
    }
    if (staged) {
      __syncwarp();
      const V* src = reinterpret_cast<const V*>(buf);
      V* dst = reinterpret_cast<V*>(a.child_rec + base * W);
      for (uint32_t v = lane; v < tt * VPR; v += 32) dst[v] = src[v];
      __syncwarp();
    }
  }
}

template <typename K>
static int launch_grid_warps(K k, const LevelArgs& a, void* stream, int smem = 0) {
  const int per_sm = cached_occupancy((const void*)k, 256, smem);
  if (per_sm < 0) return -per_sm;
  uint64_t grid = (uint64_t)cached_sm_count() * (per_sm > 0 ? per_sm : 1);
  const uint64_t need = (a.n_tiles + 7) / 8;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  k<<<(unsigned)grid, 256, smem, (cudaStream_t)stream>>>(a);
  return (int)cudaGetLastError();
}

// warp-tile levels: one wave of CTAs, never more warps than tiles
template <typename K>
static int launch_wtile_k(K k, const LevelArgs& a, void* stream) {
  const int smem = a.smem_bytes;
  const int per_sm = cached_occupancy((const void*)k, a.block, smem);
  if (per_sm < 0) return -per_sm;
  if (per_sm < 1) return (int)cudaErrorInvalidConfiguration;
  const uint64_t nw = (uint64_t)(a.block / 32);
  uint64_t grid = (uint64_t)cached_sm_count() * per_sm;
  const uint64_t need = (a.n_tiles + nw - 1) / nw;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  k<<<(unsigned)grid, a.block, smem, (cudaStream_t)stream>>>(a);
  return (int)cudaGetLastError();
}

template <int W, int CPT>
static int launch_wtile_wc(const LevelArgs& a, void* stream) {
  switch (a.hot) {
    case HOT_NONE: return launch_wtile_k(expand_wtile<W, CPT, HOT_NONE>, a, stream);
    case HOT_DIVX: return launch_wtile_k(expand_wtile<W, CPT, HOT_DIVX>, a, stream);
    case HOT_MULX: return launch_wtile_k(expand_wtile<W, CPT, HOT_MULX>, a, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

template <int W>
static int launch_nfast_emit_w(const LevelArgs& a, void* stream) {
  return launch_grid_warps(nfast_emit<W>, a, stream, 8 * kNfEmitBufBytes);  // 8 warps per block
}

template <int W>
static int launch_w(const LevelArgs& a, void* stream) {
  if (a.kind == K_NARROW) return launch_persistent(expand_narrow<W>, a, a.block, stream);
  if (a.kind == K_NFAST)
    return a.r <= 32 ? launch_grid_warps(expand_nfast<W, uint32_t>, a, stream)
                     : launch_grid_warps(expand_nfast<W, unsigned long long>, a, stream);
  if (a.kind == K_WTILE) {
    switch (a.cpt) {
      case 4: return launch_wtile_wc<W, 4>(a, stream);
      case 8: return launch_wtile_wc<W, 8>(a, stream);
      case 12: return launch_wtile_wc<W, 12>(a, stream);
      case 16: return launch_wtile_wc<W, 16>(a, stream);
      case 20: return launch_wtile_wc<W, 20>(a, stream);
      case 24: return launch_wtile_wc<W, 24>(a, stream);
      case 32: return launch_wtile_wc<W, 32>(a, stream);
      default: return (int)cudaErrorInvalidValue;
    }
  }
  switch (a.cpt) {
    case 4: return launch_wide_wc<W, 4>(a, stream);
    case 8: return launch_wide_wc<W, 8>(a, stream);
    case 16: return launch_wide_wc<W, 16>(a, stream);
    case 32: return launch_wide_wc<W, 32>(a, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

// ---------------------------------------------------------------- fused narrow tail
// The last nl levels of a group when every one is a narrow fast level (r <= 32): one
// count launch + one emit launch for all of them (atf_internal.hpp TailArgs).  The
// candidate tables of every tail level live in shared memory; a node's accept mask is
// nf_node_mask (the same exact atoms as expand_nfast), its children are its record with
// the level's field set.
struct TailTables {
  int32_t cx[kMaxTail][32];
  uint32_t cm[kMaxTail][32], ca[kMaxTail][32];
  uint32_t full[kMaxTail], nz[kMaxTail];
};

__device__ __forceinline__ void tail_stage_tables(const TailArgs& t, TailTables& S) {
  for (int i = threadIdx.x; i < kMaxTail * 32; i += blockDim.x) {
    const int d = i >> 5, c = i & 31;
    const bool v = d < t.nl && c < t.lv[d].r;
    S.cx[d][c] = v ? __ldg(t.lv[d].cand + c) : 0;
    S.cm[d][c] = v ? __ldg(t.lv[d].cand_magic + c) : 0x10000u;
    S.ca[d][c] = v ? __ldg(t.lv[d].cand_abs + c) : 0u;
  }
  __syncthreads();
  if (threadIdx.x < kMaxTail) {
    const int d = threadIdx.x;
    const int r = d < t.nl ? t.lv[d].r : 0;
    uint32_t nz = 0;
    for (int c = 0; c < r; c++) nz |= (uint32_t)(S.cx[d][c] != 0) << c;
    S.full[d] = r >= 32 ? 0xffffffffu : ((1u << r) - 1u);
    S.nz[d] = nz;
  }
  __syncthreads();
}

template <int W>
__device__ __forceinline__ void tail_child(const LevelArgs& a, const uint32_t* rec, int c, uint32_t* out) {
#pragma unroll
  for (int w = 0; w < W; w++) out[w] = rec[w] | (w == a.field_word ? (uint32_t)c << a.field_shift : 0u);
}

// subtree counts of one frontier node, depth-first (tail_count)
template <int W, int D, int NL>
__device__ __forceinline__ void tail_count_node(const TailArgs& t, const TailTables& S, const uint32_t* rec,
                                                uint32_t (&cnt)[NL]) {
  const LevelArgs& a = t.lv[D];
  uint32_t m = nf_node_mask<W, uint32_t>(a, rec, a.r, S.full[D], S.nz[D], S.cx[D], S.cm[D], S.ca[D]);
  cnt[D] += (uint32_t)__popc(m);
  if constexpr (D + 1 < NL) {
    while (m) {
      const int c = __ffs(m) - 1;
      m &= m - 1;
      uint32_t cr[W];
      tail_child<W>(a, rec, c, cr);
      tail_count_node<W, D + 1, NL>(t, S, cr, cnt);
    }
  }
}

// Pass 1: warp tile = 32 consecutive frontier nodes (lane = node); tile_total[d][tile] =
// the tile's node count at tail level d.
template <int W, int NL>
__global__ void __launch_bounds__(256, 4) tail_count(const __grid_constant__ TailArgs t) {
  __shared__ TailTables S;
  tail_stage_tables(t, S);
  const int lane = threadIdx.x & 31;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t tile = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; tile < t.n_tiles; tile += nw) {
    const uint64_t nd = tile * 32 + lane;
    uint32_t cnt[NL];
#pragma unroll
    for (int d = 0; d < NL; d++) cnt[d] = 0;
    if (nd < t.n_parents) {
      uint32_t rec[W];
      if (t.parent_rec) load_record<W>(t.parent_rec + nd * W, rec);
      else
#pragma unroll
        for (int w = 0; w < W; w++) rec[w] = 0u;
      tail_count_node<W, 0, NL>(t, S, rec, cnt);
    }
#pragma unroll
    for (int d = 0; d < NL; d++) {
      uint32_t v = cnt[d];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
      if (lane == 0) t.tile_total[(uint64_t)d * t.n_tiles + tile] = v;
    }
  }
}

// Pass 2, one tail level for a chunk of <= 32 nodes of the level above (lane = node, global
// index gidx): accept masks -> warp scan -> the chunk's CSR entries; children into the
// level's warp buffer at their chunk rank, then copied to the level's output as coalesced
// vectors at cursor[D]; then the children, in chunks of 32, are expanded one level deeper.
// Chunks are processed in node order at every depth, so every level's output is written in
// its canonical (parent-major, candidate-order) order.
template <int W, int D, int NL>
__device__ __forceinline__ void tail_emit_chunk(const TailArgs& t, const TailTables& S, const uint32_t* rec, bool valid,
                                                uint64_t gidx, uint64_t (&cursor)[NL], unsigned char* wbuf, int lane) {
  using V = typename std::conditional<W == 1, uint32_t, typename std::conditional<W == 2, uint2, uint4>::type>::type;
  constexpr int VPR = W == 8 ? 2 : 1;
  const LevelArgs& a = t.lv[D];
  uint32_t m = valid ? nf_node_mask<W, uint32_t>(a, rec, a.r, S.full[D], S.nz[D], S.cx[D], S.cm[D], S.ca[D]) : 0u;
  const uint32_t c = (uint32_t)__popc(m);
  uint32_t incl = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, incl, o);
    if (lane >= o) incl += y;
  }
  const uint32_t T = __shfl_sync(FULL, incl, 31);
  uint32_t k = incl - c;
  const uint64_t first = cursor[D];
  if (valid) t.csr[D][gidx] = first + k;
  uint32_t* buf = reinterpret_cast<uint32_t*>(wbuf + t.buf_off[D]);
  while (m) {
    const int cc = __ffs(m) - 1;
    m &= m - 1;
    uint32_t out[W];
    tail_child<W>(a, rec, cc, out);
#pragma unroll
    for (int w = 0; w < W; w++) buf[k * W + w] = out[w];
    k++;
  }
  __syncwarp();
  {
    const V* src = reinterpret_cast<const V*>(buf);
    V* dst = reinterpret_cast<V*>(t.rec[D] + first * W);
    for (uint32_t v = lane; v < T * VPR; v += 32) dst[v] = src[v];
  }
  cursor[D] = first + T;
  if constexpr (D + 1 < NL) {
    for (uint32_t s0 = 0; s0 < T; s0 += 32) {
      const bool v = s0 + lane < T;
      uint32_t cr[W];
#pragma unroll
      for (int w = 0; w < W; w++) cr[w] = v ? buf[(s0 + lane) * W + w] : 0u;
      tail_emit_chunk<W, D + 1, NL>(t, S, cr, v, first + s0 + lane, cursor, wbuf, lane);
    }
  }
  __syncwarp();  // buf[D] is refilled by the next chunk at this depth
}

template <int W, int NL>
__global__ void __launch_bounds__(32 * kTailWarps, 8) tail_emit(const __grid_constant__ TailArgs t) {
  extern __shared__ __align__(16) unsigned char tail_smem[];
  __shared__ TailTables S;
  tail_stage_tables(t, S);
  const int lane = threadIdx.x & 31;
  unsigned char* wbuf = tail_smem + (threadIdx.x >> 5) * t.warp_bytes;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw == 0 && lane < NL) {  // closing CSR entries: csr[d][size of the level above] = level total
    const uint64_t above = lane == 0 ? t.n_parents : t.tile_base[(uint64_t)(lane - 1) * (t.n_tiles + 1) + t.n_tiles];
    t.csr[lane][above] = t.tile_base[(uint64_t)lane * (t.n_tiles + 1) + t.n_tiles];
  }
  for (uint64_t tile = gw; tile < t.n_tiles; tile += nw) {
    uint64_t cursor[NL];
#pragma unroll
    for (int d = 0; d < NL; d++) cursor[d] = t.tile_base[(uint64_t)d * (t.n_tiles + 1) + tile];
    const uint64_t nd = tile * 32 + lane;
    const bool v = nd < t.n_parents;
    uint32_t rec[W];
    if (v && t.parent_rec) load_record<W>(t.parent_rec + nd * W, rec);
    else
#pragma unroll
      for (int w = 0; w < W; w++) rec[w] = 0u;
    tail_emit_chunk<W, 0, NL>(t, S, rec, v, nd, cursor, wbuf, lane);
  }
}

template <int W>
static int launch_tail_count_w(const TailArgs& t, void* stream) {
  const void* k = nullptr;
  switch (t.nl) {
    case 2: k = (const void*)tail_count<W, 2>; break;
    case 3: k = (const void*)tail_count<W, 3>; break;
    case 4: k = (const void*)tail_count<W, 4>; break;
    default: return (int)cudaErrorInvalidValue;
  }
  const int per_sm = cached_occupancy(k, 256, 0);
  if (per_sm < 0) return -per_sm;
  uint64_t grid = (uint64_t)cached_sm_count() * (per_sm > 0 ? per_sm : 1);
  const uint64_t need = (t.n_tiles + 7) / 8;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  switch (t.nl) {
    case 2: tail_count<W, 2><<<(unsigned)grid, 256, 0, (cudaStream_t)stream>>>(t); break;
    case 3: tail_count<W, 3><<<(unsigned)grid, 256, 0, (cudaStream_t)stream>>>(t); break;
    default: tail_count<W, 4><<<(unsigned)grid, 256, 0, (cudaStream_t)stream>>>(t); break;
  }
  return (int)cudaGetLastError();
}

template <int W>
static int launch_tail_emit_w(const TailArgs& t, void* stream) {
  const void* k = nullptr;
  switch (t.nl) {
    case 2: k = (const void*)tail_emit<W, 2>; break;
    case 3: k = (const void*)tail_emit<W, 3>; break;
    case 4: k = (const void*)tail_emit<W, 4>; break;
    default: return (int)cudaErrorInvalidValue;
  }
  const int smem = kTailWarps * t.warp_bytes;
  const int per_sm = cached_occupancy(k, 32 * kTailWarps, smem);
  if (per_sm < 0) return -per_sm;
  if (per_sm < 1) return (int)cudaErrorInvalidConfiguration;
  uint64_t grid = (uint64_t)cached_sm_count() * per_sm;
  const uint64_t need = (t.n_tiles + kTailWarps - 1) / kTailWarps;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  switch (t.nl) {
    case 2: tail_emit<W, 2><<<(unsigned)grid, 32 * kTailWarps, smem, (cudaStream_t)stream>>>(t); break;
    case 3: tail_emit<W, 3><<<(unsigned)grid, 32 * kTailWarps, smem, (cudaStream_t)stream>>>(t); break;
    default: tail_emit<W, 4><<<(unsigned)grid, 32 * kTailWarps, smem, (cudaStream_t)stream>>>(t); break;
  }
  return (int)cudaGetLastError();
}

}  // namespace atf
