// dev_common.cuh — device helpers shared by the sm_100a kernels: the constraint
// bytecode interpreter (SURVEY.md §8(b) semantics) and the decoupled look-back of the
// single-pass scan (tile status word = 2-bit flag + 62-bit value).
#pragma once
#include <cuda_runtime.h>
#include <cuda/atomic>
#include <stdint.h>

#include <map>
#include <mutex>
#include <tuple>

#include "atf_internal.hpp"

namespace atf {

// ---------------------------------------------------------------- host launch helpers
// Launch-configuration queries cached per process: the per-level host time sits between two
// device-idle synchronisations, so attribute / occupancy queries are paid once, not per launch.
inline int cached_sm_count() {
  static int n = 0;
  if (!n) {
    int d = 0, c = 0;
    cudaGetDevice(&d);
    cudaDeviceGetAttribute(&c, cudaDevAttrMultiProcessorCount, d);
    n = c > 0 ? c : 148;
  }
  return n;
}
// resident blocks per SM of kernel k (raises its dynamic shared-memory limit when needed);
// returns < 0 (a cudaError_t, negated) on failure
inline int cached_occupancy(const void* k, int block, int smem) {
  static std::mutex mu;
  static std::map<std::tuple<const void*, int, int>, int> occ;
  static std::map<const void*, int> smem_limit;
  std::lock_guard<std::mutex> lk(mu);
  const auto key = std::make_tuple(k, block, smem);
  auto it = occ.find(key);
  if (it != occ.end()) return it->second;
  int& lim = smem_limit[k];
  if (smem > lim) {
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return -(int)e;
    lim = smem;
  }
  int per_sm = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, block, smem);
  if (e != cudaSuccess) return -(int)e;
  occ[key] = per_sm;
  return per_sm;
}


#define FULL 0xffffffffu

// ---------------------------------------------------------------- division helpers
// 64-bit '/' and '%' compile to a called subroutine on sm_100a, and a call in a kernel
// caps its register allocation.  Operands that fit 32 bits (every C1-C5 value) take the
// inlined 32-bit path; wider ones a restoring long division (rare, call-free).
__device__ __forceinline__ uint64_t udivmod64_slow(uint64_t n, uint64_t d, uint64_t* rem) {
  uint64_t q = 0, r = 0;
  for (int i = 63; i >= 0; i--) {
    const bool carry = (r >> 63) != 0;
    r = (r << 1) | ((n >> i) & 1ull);
    if (carry || r >= d) {
      r -= d;
      q |= 1ull << i;
    }
  }
  *rem = r;
  return q;
}
__device__ __forceinline__ uint64_t udiv64f(uint64_t a, uint64_t b) {
  if (((a | b) >> 32) == 0) return (uint64_t)((uint32_t)a / (uint32_t)b);
  uint64_t r;
  return udivmod64_slow(a, b, &r);
}
__device__ __forceinline__ uint64_t umod64f(uint64_t a, uint64_t b) {
  if (((a | b) >> 32) == 0) return (uint64_t)((uint32_t)a % (uint32_t)b);
  uint64_t r;
  udivmod64_slow(a, b, &r);
  return r;
}
// signed, C truncation (quotient toward zero, remainder has the sign of a); b != 0 and
// not (a == INT64_MIN && b == -1) (the interpreter handles b == -1 before calling)
__device__ __forceinline__ int64_t sdiv64f(int64_t a, int64_t b) {
  const uint64_t ua = a < 0 ? 0ull - (uint64_t)a : (uint64_t)a, ub = b < 0 ? 0ull - (uint64_t)b : (uint64_t)b;
  const uint64_t q = udiv64f(ua, ub);
  return ((a < 0) != (b < 0)) ? (int64_t)(0ull - q) : (int64_t)q;
}
__device__ __forceinline__ int64_t smod64f(int64_t a, int64_t b) {
  const uint64_t ua = a < 0 ? 0ull - (uint64_t)a : (uint64_t)a, ub = b < 0 ? 0ull - (uint64_t)b : (uint64_t)b;
  const uint64_t r = umod64f(ua, ub);
  return a < 0 ? (int64_t)(0ull - r) : (int64_t)r;
}

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
      case 7: if (b == 0) { poison = true; r = 0; } else if (b == -1) { r = (int64_t)(0ull - (uint64_t)a); } else { r = sdiv64f(a, b); } break;
      case 8: if (b == 0) { poison = true; r = 0; } else if (b == -1) { r = 0; } else { r = smod64f(a, b); } break;
      case 9: r = a < b ? a : b; break;
      case 10: r = a > b ? a : b; break;
      case 11: r = (a == b); break;
      case 12: r = (a != b); break;
      case 13: r = (a < b); break;
      case 14: r = (a <= b); break;
      case 15: r = (a > b); break;
      case 16: r = (a >= b); break;
      case 17: if (a == 0) { poison = true; r = 0; } else if (a == -1) { r = 1; } else { r = (smod64f(b, a) == 0); } break;
      case 18: if (b == 0) { poison = true; r = 0; } else if (b == -1) { r = 1; } else { r = (smod64f(a, b) == 0); } break;
      case 19: r = (a != 0) & (b != 0); break;
      case 20: r = (a != 0) | (b != 0); break;
      default: poison = true; break;
    }
    st[sp - 1] = r;
    i += 1;
  }
  return sp == 1 ? st[0] : (poison = true, 0);
}

// q | nb for 16-bit operands (nb < 2^16, 1 <= q < 2^16) without an integer division: k =
// round(nb * rcp(q)) in fp32 (operands exact; approximate rcp within 2 ulp, so |nb/q - k| <
// 2^-6 whenever q divides nb and k is then nb / q), divisible iff k * q == nb (exact integer
// check: no false positives).
__device__ __forceinline__ bool divisible16(uint32_t nb, uint32_t q) {
  float rq;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(rq) : "f"((float)q));
  const uint32_t k = __float2uint_rn((float)nb * rq);
  return k * q == nb;
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
__device__ __forceinline__ unsigned long long lookback(unsigned long long* status, uint64_t tile, unsigned long long agg,
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

}  // namespace atf
