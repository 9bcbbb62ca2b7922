// kernels.cu — sm_100a kernels of the ATF search-space generator other than the level
// expansion (expand.cuh): the batched decoder, the standalone
// look-back scan used by the tests, and the shard offset fix-up.
#include <algorithm>

#include "dev_common.cuh"

namespace atf {

int launch_expand_w1(const LevelArgs& a, void* stream);
int launch_expand_w2(const LevelArgs& a, void* stream);
int launch_expand_w4(const LevelArgs& a, void* stream);
int launch_expand_w8(const LevelArgs& a, void* stream);
int launch_nfast_emit_w1(const LevelArgs& a, void* stream);
int launch_nfast_emit_w2(const LevelArgs& a, void* stream);
int launch_nfast_emit_w4(const LevelArgs& a, void* stream);
int launch_nfast_emit_w8(const LevelArgs& a, void* stream);

int launch_nfast_emit(const LevelArgs& a, int words, void* stream) {
  switch (words) {
    case 1: return launch_nfast_emit_w1(a, stream);
    case 2: return launch_nfast_emit_w2(a, stream);
    case 4: return launch_nfast_emit_w4(a, stream);
    case 8: return launch_nfast_emit_w8(a, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

int launch_tail_count_w1(const TailArgs& t, void* stream);
int launch_tail_count_w2(const TailArgs& t, void* stream);
int launch_tail_count_w4(const TailArgs& t, void* stream);
int launch_tail_count_w8(const TailArgs& t, void* stream);
int launch_tail_emit_w1(const TailArgs& t, void* stream);
int launch_tail_emit_w2(const TailArgs& t, void* stream);
int launch_tail_emit_w4(const TailArgs& t, void* stream);
int launch_tail_emit_w8(const TailArgs& t, void* stream);

int launch_tail_count(const TailArgs& t, int words, void* stream) {
  switch (words) {
    case 1: return launch_tail_count_w1(t, stream);
    case 2: return launch_tail_count_w2(t, stream);
    case 4: return launch_tail_count_w4(t, stream);
    case 8: return launch_tail_count_w8(t, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

int launch_tail_emit(const TailArgs& t, int words, void* stream) {
  switch (words) {
    case 1: return launch_tail_emit_w1(t, stream);
    case 2: return launch_tail_emit_w2(t, stream);
    case 4: return launch_tail_emit_w4(t, stream);
    case 8: return launch_tail_emit_w8(t, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

int launch_expand(const LevelArgs& a, int words, void* stream) {
  switch (words) {
    case 1: return launch_expand_w1(a, stream);
    case 2: return launch_expand_w2(a, stream);
    case 4: return launch_expand_w4(a, stream);
    case 8: return launch_expand_w8(a, stream);
    default: return (int)cudaErrorInvalidValue;
  }
}

int expand_smem_bytes(const LevelArgs& a, int words) { return expand_layout(a, words).total; }

// ---------------------------------------------------------------- level, second half
// After the expand kernel (every kind): tile_base = exclusive scan of the tile totals
// (scan_kernel, which also records piece_tile[p] = the tile holding output record
// p << kPieceShift).  Then (1) every parent's tile-local CSR entry gets its tile's base
// (grid-stride, coalesced) and (2) the level's records are copied from the tiles' stash
// segments to their final positions in pieces of 2^kPieceShift output records, one warp
// per piece (a piece may span several small tiles; a large tile spans many pieces), so
// the copy is balanced whatever the tile sizes.  Records move as W-word vectors, 4 loads
// in flight per lane.
template <int W>
struct RecVec;
template <> struct RecVec<1> { using T = uint32_t; };
template <> struct RecVec<2> { using T = uint2; };
template <> struct RecVec<4> { using T = uint4; };
template <> struct RecVec<8> { using T = uint4; };  // two uint4 per record

template <int W>
__global__ void __launch_bounds__(256) level_emit_kernel(const __grid_constant__ LevelArgs a) {
  using V = typename RecVec<W>::T;
  constexpr int VPR = W == 8 ? 2 : 1;  // vectors per record
  const int psh = a.piece_shift;
  const uint64_t P = 1ull << psh;
  const int lane = threadIdx.x & 31;
  const uint64_t gt = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t nt = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t total = a.tile_base[a.n_tiles];
  const bool over = total > a.child_cap || total > a.stash_cap;
  if (gt == 0) {
    if (over) atomicOr(a.overflow_flag, 1u);
    *a.total_out = total;
    a.csr[a.n_parents] = total;
  }
  // (1) CSR fix-up
  if (a.n_chunks == 1) {
    const uint64_t tn = (uint64_t)a.tile_nodes;
    if ((tn & (tn - 1)) == 0) {
      const int sh = __ffsll((long long)tn) - 1;
      for (uint64_t n = gt; n < a.n_parents; n += nt) a.csr[n] += a.tile_base[n >> sh];
    } else {
      for (uint64_t n = gt; n < a.n_parents; n += nt) a.csr[n] += a.tile_base[udiv64f(n, tn)];
    }
  } else {
    for (uint64_t n = gt; n < a.n_parents; n += nt) a.csr[n] += a.tile_base[n * (uint64_t)a.n_chunks];
  }
  if (over) return;
  // (2) pieces.  A window of 32 consecutive tiles (lane j holds tile t0 + j's base, count
  // and stash segment); each output record finds its tile by a 5-step shuffle search of
  // the window; 4 records per lane in flight.
  const uint64_t gw = gt >> 5, nw = nt >> 5;
  const uint64_t n_pieces = (total + P - 1) >> psh;
  for (uint64_t p = gw; p < n_pieces; p += nw) {
    uint64_t o = p << psh;
    const uint64_t o_end = min(o + P, total);
    uint64_t t0 = a.piece_tile[p];
    while (o < o_end) {
      const uint64_t tt = t0 + lane;
      const bool tv = tt < a.n_tiles;
      const uint64_t bj = tv ? a.tile_base[tt] : ~0ull;
      const uint64_t ej = tv ? bj + a.tile_total[tt] : ~0ull;
      const uint64_t sj = tv ? a.tile_seg[tt] : 0ull;
      // records of this window: [o, lim)
      const uint64_t e31 = __shfl_sync(FULL, ej, 31);
      const uint64_t lim = min(o_end, e31);
      for (uint64_t ob = o; ob < lim; ob += 128) {
        V v[4][VPR];
        uint64_t dsto[4];
#pragma unroll
        for (int u = 0; u < 4; u++) {
          const uint64_t oo = ob + (uint64_t)u * 32 + lane;
          int j = 0;
#pragma unroll
          for (int s = 16; s > 0; s >>= 1) {
            const uint64_t bb = __shfl_sync(FULL, bj, j + s);
            if (bb <= oo) j += s;
          }
          const uint64_t bsel = __shfl_sync(FULL, bj, j), ssel = __shfl_sync(FULL, sj, j);
          dsto[u] = oo;
          if (oo < lim) {
            const V* src = reinterpret_cast<const V*>(a.stash + (ssel + (oo - bsel)) * W);
#pragma unroll
            for (int q = 0; q < VPR; q++) v[u][q] = __ldcs(src + q);
          }
        }
#pragma unroll
        for (int u = 0; u < 4; u++)
          if (dsto[u] < lim) {
            V* dst = reinterpret_cast<V*>(a.child_rec + dsto[u] * W);
#pragma unroll
            for (int q = 0; q < VPR; q++) dst[q] = v[u][q];
          }
      }
      o = lim;
      t0 += 31;  // tile t0 + 31 holds record lim - 1 (or the window ended inside it)
      while (o < o_end && a.tile_base[t0] + a.tile_total[t0] <= o) t0++;
    }
  }
}

int launch_level_emit(const LevelArgs& a, int words, void* stream) {
  if (a.n_tiles == 0) return 0;
  const int sms = cached_sm_count();
  // enough warps for the larger of the parents (CSR) and the records (pieces); the
  // record count is only known on the device, so the grid covers the stash capacity
  const uint64_t pieces = (a.stash_cap >> a.piece_shift) + 1;
  uint64_t blocks = std::max<uint64_t>((a.n_parents + 255) / 256, (pieces + 7) / 8);
  const uint64_t cap = (uint64_t)sms * 8;
  if (blocks > cap) blocks = cap;
  if (blocks < 1) blocks = 1;
  cudaStream_t st = (cudaStream_t)stream;
  switch (words) {
    case 1: level_emit_kernel<1><<<(unsigned)blocks, 256, 0, st>>>(a); break;
    case 2: level_emit_kernel<2><<<(unsigned)blocks, 256, 0, st>>>(a); break;
    case 4: level_emit_kernel<4><<<(unsigned)blocks, 256, 0, st>>>(a); break;
    case 8: level_emit_kernel<8><<<(unsigned)blocks, 256, 0, st>>>(a); break;
    default: return (int)cudaErrorInvalidValue;
  }
  return (int)cudaGetLastError();
}

// ---------------------------------------------------------------- decode
// index -> mixed-radix digits (group 0 most significant, P:229-231 reading #11) ->
// per group: leaf record -> positions -> values; int32 SoA output, or int64 (OutT = int64_t,
// reading #22: an int64 parameter's position indexes its int64 table lvl_range64).
template <typename OutT>
__device__ __forceinline__ OutT level_value(const DecodeArgs& a, int l, uint32_t pos) {
  if constexpr (sizeof(OutT) == 8) {
    if (a.lvl_range64[l]) return __ldg(a.lvl_range64[l] + pos);
  }
  return (OutT)__ldg(a.lvl_range[l] + pos);
}
template <typename OutT>
__device__ __forceinline__ OutT bad_value() {
  if constexpr (sizeof(OutT) == 8) return (OutT)INT64_MIN;
  return (OutT)INT32_MIN;
}

template <typename OutT>
__global__ void decode_kernel(const __grid_constant__ DecodeArgs a, const uint64_t* __restrict__ idx,
                              const uint64_t* __restrict__ digits, int64_t n, OutT* __restrict__ out,
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
      for (int p = 0; p < a.n_params; p++) out[(int64_t)p * ld + i] = bad_value<OutT>();
      atomicOr(bad, 1u);
      continue;
    }
    for (int g = a.n_groups - 1; g >= 0; g--) {
      uint64_t d;
      if (idx) {  // rem / sz by multiply-high with floor((2^64-1)/sz) + at most 2 corrections
        const uint64_t sz = a.gsize[g];
        uint64_t q = __umul64hi(rem, a.gmagic[g]);
        uint64_t rr = rem - q * sz;
        while (rr >= sz) {
          q++;
          rr -= sz;
        }
        d = rr;
        rem = q;
      } else {
        d = __ldg(digits + (int64_t)g * n + i);
      }
      const int W = a.words[g];
      const uint32_t* rp = a.leaves[g] + d * (uint64_t)W;
      // record words in registers (static indices only: no local-memory array)
      uint32_t rec[8] = {0, 0, 0, 0, 0, 0, 0, 0};
      // random gather: L2 only (32-byte sectors), no 128-byte L1 line fill
      if (W == 1) {
        rec[0] = __ldcg(rp);
      } else if (W == 2) {
        const uint2 v = __ldcg(reinterpret_cast<const uint2*>(rp));
        rec[0] = v.x; rec[1] = v.y;
      } else {
        const uint4 v = __ldcg(reinterpret_cast<const uint4*>(rp));
        rec[0] = v.x; rec[1] = v.y; rec[2] = v.z; rec[3] = v.w;
        if (W == 8) {
          const uint4 u = __ldcg(reinterpret_cast<const uint4*>(rp) + 1);
          rec[4] = u.x; rec[5] = u.y; rec[6] = u.z; rec[7] = u.w;
        }
      }
      for (int l = a.lvl_begin[g]; l < a.lvl_begin[g + 1]; l++) {
        const int lw = a.lvl_word[l];
        uint32_t word = rec[0];
#pragma unroll
        for (int w = 1; w < 8; w++)
          if (lw == w) word = rec[w];
        const uint32_t bits = (uint32_t)a.lvl_bits[l];
        const uint32_t pos = bits ? (word >> a.lvl_shift[l]) & ((1u << bits) - 1u) : 0u;
        out[(int64_t)a.lvl_param[l] * ld + i] = level_value<OutT>(a, l, pos);
      }
    }
  }
}

static int launch_decode(const DecodeArgs& a, const uint64_t* idx, const uint64_t* digits, int64_t n, void* out,
                         int w64, int64_t ld, unsigned int* bad, void* stream) {
  if (n <= 0) return 0;
  uint64_t S = 1;
  int fits = 1;
  for (int g = 0; g < a.n_groups; g++) {
    const unsigned __int128 t = (unsigned __int128)S * a.gsize[g];
    if (t >> 64) fits = 0;
    S = (uint64_t)t;
  }
  const int sms = cached_sm_count();
  int64_t blocks = (n + 255) / 256;
  const int64_t cap = (int64_t)sms * 8;
  if (blocks > cap) blocks = cap;
  if (w64)
    decode_kernel<int64_t><<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(a, idx, digits, n, (int64_t*)out, ld,
                                                                                bad, S, fits);
  else
    decode_kernel<int32_t><<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(a, idx, digits, n, (int32_t*)out, ld,
                                                                                bad, S, fits);
  return (int)cudaGetLastError();
}

// Indices beyond 2^64 (S >= 2^64, P:280 mentions spaces of ~10^19): u128 index = hi * 2^64 + lo,
// either per row (idx_lo / idx_hi) or the consecutive range first + i (exhaustive search).
// Mixed radix in u128 (group 0 most significant), then the same leaf gather as decode_kernel.
template <typename OutT>
__global__ void decode128_kernel(const __grid_constant__ DecodeArgs a, const uint64_t* __restrict__ idx_lo,
                                 const uint64_t* __restrict__ idx_hi, uint64_t first_lo, uint64_t first_hi, int64_t n,
                                 OutT* __restrict__ out, int64_t ld, unsigned int* bad, uint64_t S_lo, uint64_t S_hi) {
  typedef unsigned __int128 u128;
  const u128 S = ((u128)S_hi << 64) | S_lo;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    u128 rem = idx_lo ? (((u128)__ldg(idx_hi + i) << 64) | __ldg(idx_lo + i))
                      : ((((u128)first_hi << 64) | first_lo) + (u128)i);
    if (rem >= S) {
      for (int p = 0; p < a.n_params; p++) out[(int64_t)p * ld + i] = bad_value<OutT>();
      atomicOr(bad, 1u);
      continue;
    }
    for (int g = a.n_groups - 1; g >= 0; g--) {
      const uint64_t sz = a.gsize[g];
      const u128 q = rem / sz;
      const uint64_t d = (uint64_t)(rem - q * sz);
      rem = q;
      const int W = a.words[g];
      const uint32_t* rp = a.leaves[g] + d * (uint64_t)W;
      uint32_t rec[8] = {0, 0, 0, 0, 0, 0, 0, 0};
      for (int w = 0; w < W; w++) rec[w] = __ldg(rp + w);
      for (int l = a.lvl_begin[g]; l < a.lvl_begin[g + 1]; l++) {
        const int lw = a.lvl_word[l];
        uint32_t word = rec[0];
#pragma unroll
        for (int w = 1; w < 8; w++)
          if (lw == w) word = rec[w];
        const uint32_t bits = (uint32_t)a.lvl_bits[l];
        const uint32_t pos = bits ? (word >> a.lvl_shift[l]) & ((1u << bits) - 1u) : 0u;
        out[(int64_t)a.lvl_param[l] * ld + i] = level_value<OutT>(a, l, pos);
      }
    }
  }
}

int launch_decode128(const DecodeArgs& a, const uint64_t* idx_lo, const uint64_t* idx_hi, uint64_t first_lo,
                     uint64_t first_hi, int64_t n, void* out, int w64, int64_t ld, unsigned int* bad, uint64_t S_lo,
                     uint64_t S_hi, void* stream) {
  if (n <= 0) return 0;
  const int sms = cached_sm_count();
  int64_t blocks = (n + 255) / 256;
  const int64_t cap = (int64_t)sms * 8;
  if (blocks > cap) blocks = cap;
  if (w64)
    decode128_kernel<int64_t><<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(
        a, idx_lo, idx_hi, first_lo, first_hi, n, (int64_t*)out, ld, bad, S_lo, S_hi);
  else
    decode128_kernel<int32_t><<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(
        a, idx_lo, idx_hi, first_lo, first_hi, n, (int32_t*)out, ld, bad, S_lo, S_hi);
  return (int)cudaGetLastError();
}

int launch_decode_indices(const DecodeArgs& a, const uint64_t* idx, int64_t n, void* out, int w64, int64_t ld,
                          unsigned int* bad, void* stream) {
  return launch_decode(a, idx, nullptr, n, out, w64, ld, bad, stream);
}
int launch_decode_digits(const DecodeArgs& a, const uint64_t* digits, int64_t n, void* out, int w64, int64_t ld,
                         unsigned int* bad, void* stream) {
  return launch_decode(a, nullptr, digits, n, out, w64, ld, bad, stream);
}

// ---------------------------------------------------------------- encode
// configuration (int32 SoA, column p at vals + p*ld) -> per-group digits [G][n] (UINT64_MAX:
// the row is not a valid configuration, i.e. not in the space) and, if idx != null, the
// mixed-radix index (group 0 most significant; UINT64_MAX when invalid).
// Leaf index of group g for row i (UINT64_MAX if the group's values are not a valid path).
__device__ uint64_t encode_group(const EncodeArgs& a, const int32_t* __restrict__ vals, int64_t ld, int64_t i, int g) {
  const int l0 = a.lvl_begin[g], l1 = a.lvl_begin[g + 1];
  if (l1 <= l0) return ~0ull;
  uint64_t lo = 0, hi = a.lvl_n[l0], node = 0;
  for (int l = l0; l < l1; l++) {
    const int32_t v = vals[(int64_t)a.lvl_param[l] * ld + i];
    // value -> range position
    const int32_t* sv = a.lvl_sorted[l];
    const int r = a.lvl_r[l];
    int b = 0, e = r;
    while (b < e) {
      const int m = (b + e) >> 1;
      if (__ldg(sv + m) < v) b = m + 1; else e = m;
    }
    if (b >= r || __ldg(sv + b) != v) return ~0ull;
    const uint32_t pos = (uint32_t)__ldg(sv + r + b);
    // position -> child among [lo, hi) (children sorted by their level-l field)
    const int W = a.lvl_words[l];
    const uint32_t* rec = a.lvl_rec[l] + a.lvl_word[l];
    const uint32_t bits = (uint32_t)a.lvl_bits[l];
    const uint32_t fm = bits >= 32 ? 0xffffffffu : ((1u << bits) - 1u);
    const int sh = a.lvl_shift[l];
    uint64_t cb = lo, ce = hi;
    while (cb < ce) {
      const uint64_t m = (cb + ce) >> 1;
      const uint32_t f = bits ? (__ldg(rec + m * (uint64_t)W) >> sh) & fm : 0u;
      if (f < pos) cb = m + 1; else ce = m;
    }
    if (cb >= hi || (bits ? (__ldg(rec + cb * (uint64_t)W) >> sh) & fm : 0u) != pos) return ~0ull;
    node = cb;
    if (l + 1 < l1) {
      lo = __ldg(a.lvl_csr[l] + node);
      hi = __ldg(a.lvl_csr[l] + node + 1);
    }
  }
  return node;
}

__global__ void encode_kernel(const __grid_constant__ EncodeArgs a, const int32_t* __restrict__ vals, int64_t ld,
                              int64_t n, uint64_t* __restrict__ digits, uint64_t* __restrict__ idx) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    bool ok = true;
    uint64_t index = 0;
    for (int g = 0; g < a.n_groups; g++) {
      const uint64_t d = encode_group(a, vals, ld, i, g);
      digits[(int64_t)g * n + i] = d;
      ok = ok && d != ~0ull;
      index = index * a.gsize[g] + d;
    }
    if (idx) idx[i] = ok ? index : ~0ull;
  }
}

// counter-based generator shared by nothing else: splitmix64 of (seed, row, draw)
__device__ __forceinline__ uint64_t nb_rand(uint64_t seed, uint64_t row, uint64_t k) {
  uint64_t z = seed + 0x9E3779B97F4A7C15ull * (row * 0x100000001B3ull + k + 1);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Random neighbours (simulated annealing P:217-223): row i of
// `out` = row i of `in` with one parameter re-drawn uniformly from its range, retried up
// to max_tries times until the changed row is a valid configuration (only the changed
// parameter's group is re-walked: the other groups are untouched).  moved[i] = the changed
// parameter, or -1 if no valid neighbour was found (row copied unchanged).
__global__ void neighbor_kernel(const __grid_constant__ EncodeArgs a, const int32_t* __restrict__ in, int64_t ld_in,
                                int32_t* __restrict__ out, int64_t ld_out, int64_t n, uint64_t seed, int max_tries,
                                int32_t* __restrict__ moved) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    for (int p = 0; p < a.n_params; p++) out[(int64_t)p * ld_out + i] = in[(int64_t)p * ld_in + i];
    int32_t mv = -1;
    for (int t = 0; t < max_tries && mv < 0; t++) {
      const uint64_t r1 = nb_rand(seed, (uint64_t)i, 2 * (uint64_t)t), r2 = nb_rand(seed, (uint64_t)i, 2 * (uint64_t)t + 1);
      const int p = (int)(r1 % (uint64_t)a.n_params);
      const int rp = a.param_r[p];
      if (rp <= 1) continue;
      const int32_t old = out[(int64_t)p * ld_out + i];
      const int32_t v = __ldg(a.param_range[p] + (int64_t)(r2 % (uint64_t)rp));
      if (v == old) continue;
      out[(int64_t)p * ld_out + i] = v;
      if (encode_group(a, out, ld_out, i, a.param_group[p]) != ~0ull) mv = p;
      else out[(int64_t)p * ld_out + i] = old;
    }
    moved[i] = mv;
  }
}

int launch_neighbors(const EncodeArgs& a, const int32_t* in, int64_t ld_in, int32_t* out, int64_t ld_out, int64_t n,
                     uint64_t seed, int max_tries, int32_t* moved, void* stream) {
  if (n <= 0) return 0;
  const int sms = cached_sm_count();
  int64_t blocks = (n + 255) / 256;
  if (blocks > (int64_t)sms * 8) blocks = (int64_t)sms * 8;
  neighbor_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(a, in, ld_in, out, ld_out, n, seed, max_tries,
                                                                        moved);
  return (int)cudaGetLastError();
}

int launch_encode(const EncodeArgs& a, const int32_t* vals, int64_t ld, int64_t n, uint64_t* digits, uint64_t* idx,
                  void* stream) {
  if (n <= 0) return 0;
  const int sms = cached_sm_count();
  int64_t blocks = (n + 255) / 256;
  if (blocks > (int64_t)sms * 8) blocks = (int64_t)sms * 8;
  encode_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(a, vals, ld, n, digits, idx);
  return (int)cudaGetLastError();
}

// ---------------------------------------------------------------- CLTune-style baseline
// Thread t takes tuples [t*chunk, (t+1)*chunk) of the full product in declaration order
// (last parameter fastest): one mixed-radix decode of its first tuple, then an odometer.
// A tuple is valid iff every parameter's constraint holds (strict bytecode semantics; a
// tuple is rejected at its first failing parameter).  Valid tuples are counted.
__global__ void filter_product_kernel(const __grid_constant__ ProductArgs a, unsigned long long* count) {
  const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t b = t * a.chunk;
  unsigned long long ok = 0;
  if (b < a.total) {
    const uint64_t e = min(b + a.chunk, a.total);
    const int P = a.n_params;
    int32_t pos[kMaxLevels];
    int64_t val[kMaxLevels];
    uint64_t rem = b;
    for (int p = P - 1; p >= 0; p--) {
      const uint64_t rp = (uint64_t)a.r[p];
      pos[p] = (int32_t)(rem % rp);
      rem /= rp;
      val[p] = __ldg(a.range[p] + pos[p]);
    }
    for (uint64_t i = b; i < e; i++) {
      bool good = true;
      for (int p = 0; p < P && good; p++) {
        for (int q = a.prog_first[p]; q < a.prog_first[p] + a.prog_count[p] && good; q++) {  // ANDed
          bool poison = false;
          const int64_t v = run_code(a.code + __ldg(a.progs + 2 * q), __ldg(a.progs + 2 * q + 1), val[p], val, 1, poison);
          good = !poison && v != 0;
        }
      }
      ok += good;
      for (int p = P - 1; p >= 0; p--) {  // odometer
        if (++pos[p] < a.r[p]) {
          val[p] = __ldg(a.range[p] + pos[p]);
          break;
        }
        pos[p] = 0;
        val[p] = __ldg(a.range[p]);
      }
    }
  }
  ok = warp_sum_u64(ok);
  if ((threadIdx.x & 31) == 0 && ok) atomicAdd(count, ok);
}

int launch_filter_product(const ProductArgs& a, unsigned long long* count, void* stream) {
  if (a.total == 0) return 0;
  const uint64_t threads = (a.total + a.chunk - 1) / a.chunk;
  const uint64_t blocks = (threads + 255) / 256;
  if (blocks > 0x7fffffffull) return (int)cudaErrorInvalidValue;
  filter_product_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(a, count);
  return (int)cudaGetLastError();
}

// ---------------------------------------------------------------- divisible16 check (tests)
// Exhaustive: every (nb, q) with nb < 2^16, 1 <= q < 2^16 against integer modulo.
__global__ void divisible16_check_kernel(unsigned long long* mismatches) {
  unsigned long long bad = 0;
  for (uint32_t q = blockIdx.x + 1; q < 65536u; q += gridDim.x)
    for (uint32_t nb = threadIdx.x; nb < 65536u; nb += blockDim.x) bad += divisible16(nb, q) != (nb % q == 0);
  bad = warp_sum_u64(bad);
  if ((threadIdx.x & 31) == 0 && bad) atomicAdd(mismatches, bad);
}
int launch_divisible16_check(unsigned long long* mismatches, void* stream) {
  divisible16_check_kernel<<<4096, 256, 0, (cudaStream_t)stream>>>(mismatches);
  return (int)cudaGetLastError();
}

// ---------------------------------------------------------------- standalone scan (tests)
// Exclusive scan u32 -> u64 with the same look-back as expand_kernel; out[n] = total.
// blockIdx.y selects one of several independent scans of equal length (the fused tail's levels):
// arrays at in + y * n, out + y * (n + 1), status + y * st_stride, counter + y.
__global__ void scan_kernel(const uint32_t* __restrict__ in, uint64_t* __restrict__ out, int64_t n,
                            unsigned long long* status, unsigned int* counter, uint64_t n_tiles,
                            uint32_t* __restrict__ piece_tile, uint64_t piece_cap, int psh, uint64_t st_stride) {
  in += (uint64_t)blockIdx.y * (uint64_t)n;
  out += (uint64_t)blockIdx.y * (uint64_t)(n + 1);
  status += (uint64_t)blockIdx.y * st_stride;
  counter += blockIdx.y;
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
      if (i0 + q < n) {
        out[i0 + q] = run;
        if (piece_tile && v[q]) {  // pieces whose first record lies in element i0 + q
          const uint64_t P = 1ull << psh;
          for (uint64_t p = (run + P - 1) >> psh; (p << psh) < run + v[q] && p < piece_cap; p++)
            piece_tile[p] = (uint32_t)(i0 + q);
        }
      }
      run += v[q];
    }
    __syncthreads();
  }
}

int launch_scan_u32(const uint32_t* in, uint64_t* out, int64_t n, unsigned long long* status, unsigned int* counter,
                    void* stream, uint32_t* piece_tile, uint64_t piece_cap, int piece_shift) {
  const int B = 256;
  const uint64_t n_tiles = n > 0 ? (uint64_t)((n + B * 4 - 1) / (B * 4)) : 1;
  const int sms = cached_sm_count();
  uint64_t grid = (uint64_t)sms * 4;
  if (grid > n_tiles) grid = n_tiles;
  scan_kernel<<<(unsigned)grid, B, 0, (cudaStream_t)stream>>>(in, out, n, status, counter, n_tiles, piece_tile, piece_cap,
                                                                 piece_shift, 0);
  return (int)cudaGetLastError();
}
int launch_scan_u32_batch(const uint32_t* in, uint64_t* out, int64_t n, int batch, unsigned long long* status,
                          uint64_t status_stride, unsigned int* counter, void* stream) {
  const int B = 256;
  const uint64_t n_tiles = n > 0 ? (uint64_t)((n + B * 4 - 1) / (B * 4)) : 1;
  const int sms = cached_sm_count();
  uint64_t grid = (uint64_t)sms * 4;
  if (grid > n_tiles) grid = n_tiles;
  scan_kernel<<<dim3((unsigned)grid, (unsigned)batch), B, 0, (cudaStream_t)stream>>>(
      in, out, n, status, counter, n_tiles, nullptr, 0, kPieceShift, status_stride);
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

// ---- cross-rank round flags of the replayed balanced multi-GPU generation:
// the owner publishes "round r of generation `epoch` is complete" after the round's kernels
// (stream order) with a system-scope release; a consumer's stream spins on the owner's flag
// (peer memory) with an acquire before copying the owner's records.  A wait that does not see
// the flag within ~2 s gives up and raises `err` (the generation then fails its checks and is
// regenerated with the synchronous protocol) instead of hanging the device.
__global__ void dist_flag_set_kernel(unsigned long long* f, unsigned long long v) {
  __threadfence_system();
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(v) : "memory");
}
__global__ void dist_flag_wait_kernel(const unsigned long long* f, unsigned long long v, unsigned long long* err) {
  unsigned long long t0, t, x;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(x) : "l"(f) : "memory");
    if (x >= v) return;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 2000000000ull) {
      atomicExch(err, 1ull);
      return;
    }
    __nanosleep(200);
  }
}
// Host-released gate (the balanced generation's round timing, ATF_FLAG_TIMING): the stream
// holds until the host writes `v` to the mapped word, so a round's launches are all queued
// before the device starts it and its CUDA events measure device work only (as in the replay,
// where the host runs ahead).  100 ms time-out.
__global__ void host_gate_kernel(const volatile unsigned int* flag, unsigned int v) {
  unsigned long long t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  while (*flag < v) {
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 100000000ull) return;  // 100 ms: a host call that synchronises while the gate is held
    __nanosleep(100);
  }
}
int launch_host_gate(const unsigned int* flag, unsigned int v, void* stream) {
  host_gate_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(flag, v);
  return (int)cudaGetLastError();
}
int launch_dist_flag_set(unsigned long long* f, unsigned long long v, void* stream) {
  dist_flag_set_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(f, v);
  return (int)cudaGetLastError();
}
int launch_dist_flag_wait(const unsigned long long* f, unsigned long long v, unsigned long long* err, void* stream) {
  dist_flag_wait_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(f, v, err);
  return (int)cudaGetLastError();
}

}  // namespace atf
