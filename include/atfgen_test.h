/*
 * atfgen_test.h — test hooks of libatfgen (not part of the product API).
 *
 * atf_test_exclusive_scan_u32: the decoupled look-back exclusive scan used by the
 * fused expand kernel, exposed alone so it can be checked
 * against std::exclusive_scan on adversarial count arrays.
 *   d_in:  device uint32[n]; d_out: device uint64[n + 1]; d_out[n] = total.
 *   Scratch is allocated internally (cudaMallocAsync on `stream`).  Synchronous.
 *
 * atf_test_shard_slice / atf_test_shard_offsets: the host logic of the multi-GPU shard
 * layer (atf_space_generate_shard / atf_space_finalize_shard use the
 * same functions), callable without a GPU.
 *   shard_slice:   h_csr[0..ncut] (host) = child-count prefix of the cut level; writes the
 *                  rank's contiguous slice [*lo, *hi) balanced by children.
 *   shard_offsets: h_all[world][n] (host, rank-major) per-rank counts; writes, per entry,
 *                  before[i] = sum over ranks < rank and tot[i] = sum over all ranks.
 */
#ifndef ATFGEN_TEST_H
#define ATFGEN_TEST_H
#include "atfgen.h"
#ifdef __cplusplus
extern "C" {
#endif
atf_status atf_test_exclusive_scan_u32(const uint32_t* d_in, uint64_t* d_out, int64_t n, void* stream);
atf_status atf_test_shard_slice(const uint64_t* h_csr, uint64_t ncut, int32_t rank, int32_t world, uint64_t* lo,
                                uint64_t* hi);
atf_status atf_test_shard_offsets(const int64_t* h_all, int32_t world, int32_t n, int32_t rank, uint64_t* before,
                                  uint64_t* tot);

/* Exhaustive device check of the float-reciprocal divisibility test used for 16-bit quotient
 * divisors (dev_common.cuh divisible16) against integer modulo: *h_mismatches must be 0. */
atf_status atf_test_divisible16(uint64_t* h_mismatches);
/* Source text of the NVRTC-specialised kernel of level k of group g: the pass-1 kernel of a
 * narrow fast level, the exact-mask kernel of a mid-width (32 < r <= 1024) nf_ok level; empty
 * otherwise.  Plans the space if needed.  Host only. */
atf_status atf_test_jit_source(atf_space* s, int32_t g, int32_t k, char* buf, size_t cap, size_t* len_out);
/* Source text of the NVRTC-specialised fused-tail kernels of group g (atf_tail_count +
 * atf_tail_emit; empty when the group has no fused narrow tail); plans the space.  Host only.
 * *k0_out (optional) = the tail's first level (-1 if none). */
atf_status atf_test_tail_source(atf_space* s, int32_t g, char* buf, size_t cap, size_t* len_out, int32_t* k0_out);
/* Staging bytes per warp of the fused tail's emit kernel for spaces planned afterwards (tuning
 * experiments; 0 restores the default -- 12 KB when the tail's first level has more than 32
 * candidates, else 8 KB --, a multiple of 16 in [2048, 49152] otherwise). */
atf_status atf_test_set_tail_stage(int32_t bytes);
/* Product-structured fused tails (every term of every tail level reads only ancestors above the
 * tail: the subtree under a frontier node is a grid of the levels' masks): on (1,
 * default) or off (0, the depth-first kernels) for tails compiled afterwards. */
atf_status atf_test_set_tail_product(int32_t on);
/* Fresh spaces with several groups: per-group level rounds without a barrier (1, default) or one
 * synchronising round for all groups (0).  A/B experiments. */
atf_status atf_test_set_async_rounds(int32_t on);
/* Fused-tail emit: the balanced leaf pass writes the leaves to global memory (1) or to the warp's
 * staging area (0); 2 (default): to global memory when the tail's first level has more than 32
 * candidates.  A/B experiments. */
atf_status atf_test_set_tail_leaf_direct(int32_t mode);
/* Mid-width exact-mask kernel (atf_wide_jit): candidates per superset group of the first conjunct
 * (2, 4 = default, 8, 16; 0 restores 4), for kernels compiled afterwards.  A/B experiments. */
atf_status atf_test_set_wide_group(int32_t n);
/* Geometry knobs for spaces planned / generated afterwards (tuning experiments; 0 = default):
 * warp tiles per SM below which the warp-tile kernel halves its nodes per tile (256), and
 * log2 of the candidate-pair count below which generate_dist replicates a level (28). */
atf_status atf_test_set_geometry(int32_t tiles_per_sm, int32_t repl_log2);
/* Warp-tile levels of at most n tiles are written in place behind a decoupled look-back (one
 * launch, no scan / copy kernels); 0 restores the default 16.  Tuning experiments. */
atf_status atf_test_set_direct_tiles(int32_t n);
#ifdef __cplusplus
}
#endif
#endif
