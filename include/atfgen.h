/*
 * atfgen.h — C ABI of the B200-native ATF search-space generator.
 *
 * The operation (PAPER.md, cited as P:n = line n):
 *   A tuning parameter has a unique name, a range and a constraint (P:51-59,
 *   §II Step 1).  The search space "comprises all valid parameter
 *   configurations, i.e., for which the parameters' constraints are
 *   satisfied".  ATF generates it "by iterating over the constrained
 *   ranges of tuning parameters" rather than filtering the unconstrained
 *   product, per group of interdependent parameters.
 *   The space has a size S and is index-addressable: OpenTuner's
 *   TP in [1,S] selects "the configuration with index TP within the ATF search
 *   space".
 *
 * This library builds each parameter group's valid configurations on one GPU
 * (sm_100a) as a per-level tree (level k = the group's k-th parameter), and
 * exposes S (u128), per-group sizes and a batched index -> configuration
 * decoder.  Groups are found automatically (connected components of the
 * constraint-reference graph) instead of the paper's user-supplied G(...)
 * (P:245).
 *
 * Conventions:
 *   - Indices are 0-based (the paper's TP is 1-based).
 *   - Group order: by first-declared member; group 0 is the most significant
 *     mixed-radix digit.  Inside a group: lexicographic order of range
 *     positions in declaration order.  Output columns are in declaration order.
 *   - Intervals are inclusive, value(i) = gen(begin + i*step).
 *   - A zero divisor anywhere in a constraint rejects the candidate; AND/OR
 *     are strict (non-short-circuit) (reading #7).
 *
 * Errors: every function returns atf_status (0 = ATF_OK, < 0 = error); no
 * exceptions cross the ABI.  atf_space_last_error() gives a message.
 * Threading: an atf_space is not thread-safe; distinct spaces are independent.
 * Ownership: host inputs (names, range values, bytecode) are copied before the
 * call returns.  Device buffers passed to decode are borrowed until the work
 * queued on `stream` completes.  The space owns its tree memory.
 */
#ifndef ATFGEN_H
#define ATFGEN_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct atf_space atf_space; /* opaque, owned by the library */

typedef enum {
  ATF_OK = 0,
  ATF_ERR_INVALID_ARG = -1, /* NULL pointer, bad kind, step <= 0, empty name, ...      */
  ATF_ERR_OOM = -2,         /* allocation failed (device or host)                      */
  ATF_ERR_CUDA = -3,        /* a CUDA runtime call failed (message in last_error)      */
  ATF_ERR_STATE = -4,       /* call not allowed in the space's current state           */
  ATF_ERR_BYTECODE = -5,    /* bad opcode, stack underflow/overflow, not 1 result       */
  ATF_ERR_FORWARD_REF = -6, /* PARAM j with j >= the constrained parameter's id       */
  ATF_ERR_OVERFLOW = -7,    /* int64 overflow possible / size or index too large      */
  ATF_ERR_INDEX = -8,       /* decode index >= S (rows filled with INT32_MIN)          */
  ATF_ERR_DUPLICATE = -9,   /* duplicate parameter name or duplicate set value        */
  ATF_ERR_LIMIT = -10       /* a documented v1 limit is exceeded                       */
} atf_status;

/* Range kinds ("a range of values of an arbitrary fundamental type T (e.g., bool,
 * integer, or float)").  Values are int64 (reading #22); a space whose values all fit int32
 * is an "int32 space" (decoded by the int32 entry points), otherwise an "int64 space"
 * (atf_space_value_bits() == 64; decoded by the *_i64 entry points).
 *   INTERVAL: values begin, begin+step, ..., <= end (inclusive, reading #1), any int64.
 *   POW2:     values 2^i for i = begin, begin+step, ..., <= end; 0 <= i <= 62
 *             ("atf::interval<size_t>(1,10,[](i){return pow(2,i);})" = first ten powers of 2).
 *   SET:      values[0..n_values) (int32) in the listed order; duplicates -> ATF_ERR_DUPLICATE.
 *             bool and enum parameters are SETs of ints ({0,1} for bools).
 *   GEN:      the general generator of P:57 ("the elements generator(i) for each i from
 *             begin to end"): values gen(i) for i = begin, begin+step, ..., <= end, where
 *             gen is a bytecode program (`values` = its int32 words, `n_values` = their
 *             number) in which X is i (PARAM is not allowed).  Evaluated exactly in int64
 *             on the host when the parameter is added; a poisoned value or int64 overflow ->
 *             ATF_ERR_BYTECODE / ATF_ERR_OVERFLOW, a repeated value -> ATF_ERR_DUPLICATE
 *             (reading #5).
 *   SET64:    values64[0..n_values) (int64) in the listed order; duplicates -> ATF_ERR_DUPLICATE.
 * A parameter whose values do not all fit int32 is expanded by the generic kernels (every
 * conjunct of its own level interpreted in int64; the levels that reference it read its int64
 * value table); int32 parameters keep every fast path. */
typedef enum {
  ATF_RANGE_INTERVAL = 0, ATF_RANGE_POW2 = 1, ATF_RANGE_SET = 2, ATF_RANGE_GEN = 3, ATF_RANGE_SET64 = 4
} atf_range_kind;

typedef struct {
  int32_t kind;             /* atf_range_kind */
  int64_t begin, end, step;
  const int32_t* values;    /* SET / GEN: host pointer, copied */
  int64_t n_values;         /* SET / GEN / SET64: number of entries */
  const int64_t* values64;  /* SET64 only: host pointer, copied */
} atf_range;

/* Device allocator hooks (e.g. PyTorch's caching allocator).  If alloc is NULL
 * the library uses cudaMallocAsync/cudaFreeAsync on its stream.  `stream` is the
 * cudaStream_t the memory will be used on. */
typedef void* (*atf_alloc_fn)(size_t bytes, void* stream, void* ctx);
typedef void (*atf_free_fn)(void* ptr, size_t bytes, void* stream, void* ctx);

typedef struct {
  int32_t device;      /* CUDA device ordinal                                  */
  void* stream;        /* cudaStream_t for all work (NULL = legacy default)    */
  atf_alloc_fn alloc;  /* optional */
  atf_free_fn free;    /* optional (required if alloc is set) */
  void* alloc_ctx;
  uint32_t flags;      /* ATF_FLAG_* */
} atf_space_opts;

#define ATF_FLAG_TIMING 1u        /* record per-level CUDA-event times (atf_space_stats)  */
#define ATF_FLAG_GENERIC_ONLY 2u  /* disable the hoisted fast atoms: interpret every
                                     candidate with the generic bytecode interpreter     */
#define ATF_FLAG_LEGACY_WIDE 8u   /* levels with r > 64 use the block-tile kernel instead of
                                     the warp-tile kernel (kept for parity coverage)      */
#define ATF_FLAG_NO_JIT 16u       /* narrow fast levels use the generic kernel instead of the
                                     NVRTC-specialised one (kept for parity coverage)     */
#define ATF_FLAG_SERIAL_GROUPS 32u /* run the groups' levels one after another on the space's
                                     stream (default: concurrently, one stream per group) —
                                     isolates per-launch times for roofline measurements    */
#define ATF_FLAG_KEEP_LEVELS 4u   /* keep inner-level arrays (CSR + records); default
                                     keeps them too — reserved                          */
#define ATF_FLAG_NO_SEG_BOUNDS 64u /* evaluate EVERY (frontier node, candidate) pair, i.e. all
                                     f_{k-1} * r_k candidate evaluations of the spec as written
                                     ("must not skip candidates"; P:280
                                     "iterating over the constrained ranges").  Without it the
                                     warp-tile kernel rejects whole candidate segments of a
                                     divisibility filter by their |x| bounds (x | n needs
                                     |x| <= |n|) without evaluating their pairs; the result is
                                     identical, the evaluated-pair count is not */
#define ATF_FLAG_NO_REPLAY 256u  /* every generation sizes its levels one round at a time (a host
                                     synchronisation per level round) instead of replaying the
                                     previous generation's level sizes (one synchronisation,
                                     totals verified; DESIGN.md §5 "Steady state")              */
#define ATF_FLAG_DIST_SUBSETS 512u /* (the default since round 2; kept for compatibility) */
#define ATF_FLAG_DIST_NO_SUBSETS 1024u /* atf_space_generate_dist: every group on every rank in every
                                     generation.  By default, from the second generation on, each
                                     group works on a subset of the ranks in proportion to its
                                     candidate pairs in the previous generation (DESIGN.md §6:
                                     fewer, larger kernels per rank; one-GPU steady-state
                                     prediction for C5 at N = 4 / 8: 5.2 / 3.4-3.6 ms vs
                                     5.4 / 3.75 ms) */
#define ATF_FLAG_NO_TAIL 128u     /* expand a group's trailing narrow levels one at a time instead
                                     of the fused narrow tail (two launches for up to 4 levels,
                                     DESIGN.md §5); kept for parity coverage and A/B timing    */

/* Bytecode: postfix int32 words, int64 stack.
 *   1 X            push the candidate value
 *   2 PARAM j      push the value of parameter j (j < the constrained parameter's id)
 *   3 CONST lo hi  push the int64 (hi << 32) | (uint32)lo
 *   4 ADD 5 SUB 6 MUL            exact; possible int64 overflow -> ATF_ERR_OVERFLOW
 *   7 DIV 8 MOD                  C truncation; b == 0 -> poison
 *   9 MIN 10 MAX
 *  11 EQ 12 NE 13 LT 14 LE 15 GT 16 GE   -> 0/1
 *  17 DIVIDES  a b -> [b mod a == 0]; a == 0 -> poison     (atf::divides)
 *  18 MULOF    a b -> [a mod b == 0]; b == 0 -> poison     (atf::is_multiple_of)
 *  19 AND 20 OR (strict)  21 NOT
 * A candidate is accepted iff the program leaves exactly one item, it is
 * nonzero, and no poison occurred.  Several constraints on one parameter are
 * ANDed.  Limits: <= 256 words and stack depth <= 16 per program. */
enum {
  ATF_OP_X = 1, ATF_OP_PARAM = 2, ATF_OP_CONST = 3, ATF_OP_ADD = 4, ATF_OP_SUB = 5, ATF_OP_MUL = 6,
  ATF_OP_DIV = 7, ATF_OP_MOD = 8, ATF_OP_MIN = 9, ATF_OP_MAX = 10, ATF_OP_EQ = 11, ATF_OP_NE = 12,
  ATF_OP_LT = 13, ATF_OP_LE = 14, ATF_OP_GT = 15, ATF_OP_GE = 16, ATF_OP_DIVIDES = 17,
  ATF_OP_MULOF = 18, ATF_OP_AND = 19, ATF_OP_OR = 20, ATF_OP_NOT = 21
};

/* v1 limits */
#define ATF_MAX_PARAMS 64
#define ATF_MAX_RANGE (1 << 24)
#define ATF_MAX_PROGRAM_WORDS 256
#define ATF_MAX_STACK 16

/* ---- building (state BUILDING) --------------------------------------------------- */

/* Create an empty space.  opts may be NULL (device 0, default stream).  No CUDA
 * work happens until atf_space_generate. */
atf_status atf_space_create(const atf_space_opts* opts, atf_space** out);

/* Add tuning parameter `name` (unique) with `range`.  The
 * parameter id (declaration index) is written to *out_param_id. */
atf_status atf_space_add_param(atf_space* s, const char* name, const atf_range* range,
                               int32_t* out_param_id);

/* Add a constraint program to parameter `param_id` (a callable on the
 * parameter's value that may use earlier parameters).  Validated immediately
 * (opcodes, stack discipline, backward references). */
atf_status atf_space_add_constraint(atf_space* s, int32_t param_id, const int32_t* code,
                                    int32_t n_words);

/* ---- planning (host only; no GPU needed) ----------------------------------------- */

/* Materialise ranges, run the static int64 interval analysis, partition the
 * parameters into groups and compile each level's constraint program.
 * BUILDING -> PLANNED.  Called implicitly by generate. */
atf_status atf_space_plan(atf_space* s);

atf_status atf_space_num_params(const atf_space* s, int32_t* out);
/* Name of parameter p (NUL-terminated, truncated to cap - 1 bytes); *len_out (optional) = its
 * full length.  ATF_ERR_INVALID_ARG for a bad p. */
atf_status atf_space_param_name(const atf_space* s, int32_t p, char* buf, size_t cap, size_t* len_out);
atf_status atf_space_num_groups(const atf_space* s, int32_t* out);           /* >= PLANNED */
/* members of group g (declaration order) -> out[0..n), n written to *n_out */
atf_status atf_space_group_members(const atf_space* s, int32_t g, int32_t* out, int32_t cap,
                                   int32_t* n_out);
/* JSON description of the plan (groups, levels, record layout, compiled terms). */
atf_status atf_space_plan_json(const atf_space* s, char* buf, size_t cap, size_t* len_out);

/* ---- generation (GPU) ------------------------------------------------------------- */

/* Generate every group's tree on the space's device/stream.  PLANNED (or
 * BUILDING) -> GENERATED.  Synchronises the stream once per level round. */
atf_status atf_space_generate(atf_space* s);

/* Multi-GPU: generate this rank's shard (levels above the cut replicated, a
 * contiguous balanced slice of the cut level expanded locally).  Writes this
 * rank's per-level node counts (sum over groups of their level counts, in
 * (group, level) order) to h_counts[0..n) (host), *n_out = n.  The caller
 * all-gathers the counts across ranks (e.g. NCCL over NVLink) and passes them
 * to atf_space_finalize_shard.  -> SHARDED. */
atf_status atf_space_generate_shard(atf_space* s, int32_t rank, int32_t world, int64_t* h_counts,
                                    int32_t cap, int32_t* n_out);
/* h_all_counts: [world][n] host array of every rank's counts (rank-major).
 * Computes the global level offsets of this rank's slice and the global group
 * sizes.  SHARDED -> GENERATED (size/group_size become global; decode is not
 * available on a shard: ATF_ERR_STATE). */
atf_status atf_space_finalize_shard(atf_space* s, const int64_t* h_all_counts, int32_t world,
                                    int32_t n);

/* Multi-GPU, balanced per level: called by every rank
 * (one process per GPU, or several spaces of one process).  Every level is redistributed: rank
 * r expands the parents [r F / N, (r + 1) F / N) of the previous level (F = its global size),
 * so each rank evaluates f_{k-1} r_k / N candidate pairs per level however unbalanced the tree.
 * After each level round the library calls `allgather` once: it must copy `bytes` from `send`
 * (host memory) of every rank into recv + rank * bytes on every rank and return 0 (e.g.
 * torch.distributed.all_gather_into_tensor over NCCL).  The record holds the level counts and
 * where the new level's records live; the next parent slice is then copied from the owning ranks
 * (CUDA IPC over NVLink / NVSwitch; plain device pointers between spaces of one process).  In
 * this mode the space allocates its arenas with cudaMalloc (exportable), not the allocator hooks.
 * -> state FINAL_SHARD: size / group_size / level_size global-local as after finalize_shard;
 * level_view gives this rank's slice of every level (offset, csr_offset).  Every rank must call
 * with the same spec; errors are local (a failing rank makes the others fail in the callback). */
typedef int (*atf_allgather_fn)(const void* send, void* recv, size_t bytes, void* ctx);
atf_status atf_space_generate_dist(atf_space* s, int32_t rank, int32_t world, atf_allgather_fn allgather, void* ctx);
/* Steady state of atf_space_generate_dist (like the single-GPU replay): the
 * space logs every round's all-gathered records.  The next call with the same rank, world and
 * flags sizes every level from the log (its allocations -- hence the addresses peers read --
 * are then those the replay reproduces); if every count matched, later calls queue all rounds
 * with no host synchronisation and no all-gather per round: each rank marks a finished round in
 * a device flag array (exported by CUDA IPC) and its stream waits on the owners' flags before a
 * peer copy.  One synchronisation and ONE all-gather of 4-byte verdicts per call then check
 * every level total, overflow flag, wait time-out and address against the log on every rank; a
 * failed check regenerates with the synchronous protocol in the same call.  Not used with
 * ATF_FLAG_NO_REPLAY or ATF_FLAG_TIMING.  Ranks sharing one device must use different streams
 * (a wait on the legacy default stream would block the owner's work until its 2 s time-out).
 *
 * atf_space_dist_round_ms: with ATF_FLAG_TIMING, the device time of each round of this rank's
 * last atf_space_generate_dist (CUDA events on the space's stream around the round's kernels,
 * CSR fix-ups and peer copies), out[0..n) (host), *n_out = rounds; ATF_ERR_STATE without them. */
atf_status atf_space_dist_round_ms(const atf_space* s, float* out, int32_t cap, int32_t* n_out);

/* ---- results (state GENERATED) ---------------------------------------------------- */

/* S = prod_g |G_g| as u128: *lo = low 64 bits, *hi = high 64 bits. */
atf_status atf_space_size(const atf_space* s, uint64_t* lo, uint64_t* hi);
atf_status atf_space_group_size(const atf_space* s, int32_t g, uint64_t* out);
atf_status atf_space_num_levels(const atf_space* s, int32_t g, int32_t* out);
/* f_k of group g (nodes at level k = 0..L-1, dead ends included); for a shard:
 * this rank's local count. */
atf_status atf_space_level_size(const atf_space* s, int32_t g, int32_t k, uint64_t* out);

/* Level arrays of group g, level k (device pointers owned by the space):
 *   records: [f_k][words] uint32, the range positions of the node's path
 *            (field k' at bits [shift_k', shift_k'+bits_k') of word word_k');
 *   csr:     [f_k + 1] uint64 first-child index in level k+1 (NULL for the leaf level);
 *   offset:  global index of this array's first node (0 on one GPU). */
typedef struct {
  const uint32_t* records;
  const uint64_t* csr;
  uint64_t n_nodes;
  uint64_t offset;
  int32_t words;
  int32_t param;     /* parameter id of level k */
  int32_t field_word, field_shift, field_bits;
  uint64_t csr_offset;  /* global index of the level-k node whose entry is csr[0]          */
  uint64_t csr_nodes;   /* level-k nodes the csr array covers (csr has csr_nodes + 1 entries;
                           = n_nodes / offset except after atf_space_generate_dist, where a
                           rank's CSR covers the parent slice it expanded)                   */
} atf_level_view;
atf_status atf_space_level_view(const atf_space* s, int32_t g, int32_t k, atf_level_view* out);

/* Decode n 0-based indices (device uint64 d_idx[n], requires S < 2^64 else
 * ATF_ERR_OVERFLOW) into configurations: d_out is int32 SoA, column p (the
 * value of parameter p) at d_out + p*ld, ld >= n.  Rows whose index >= S are
 * filled with INT32_MIN and the call returns ATF_ERR_INDEX (after a stream sync).
 * Otherwise asynchronous on `stream` (NULL = the space's stream).  The int32 decoders
 * (decode_indices / decode_digits / decode_indices128 / decode_range) return
 * ATF_ERR_OVERFLOW on an int64 space (reading #22): use the *_i64 decoders below. */
atf_status atf_space_decode_indices(const atf_space* s, const uint64_t* d_idx, int64_t n,
                                    int32_t* d_out, int64_t ld, void* stream);
/* Like decode_indices but with per-group digits: d_digits is [G][n] uint64
 * (digit of group g at d_digits + g*n, each < |G_g|); works for any S. */
atf_status atf_space_decode_digits(const atf_space* s, const uint64_t* d_digits, int64_t n,
                                   int32_t* d_out, int64_t ld, void* stream);

/* Indices of any size (S may be >= 2^64; P:280 mentions spaces of ~10^19 configurations):
 * index i = hi * 2^64 + lo.  decode_indices128 takes per-row device arrays d_idx_lo[n] /
 * d_idx_hi[n]; decode_range decodes the n consecutive indices first, first + 1, ... (the
 * exhaustive search of P:218) with first = first_hi * 2^64 + first_lo.  Output and errors as
 * atf_space_decode_indices (rows >= S: INT32_MIN and ATF_ERR_INDEX; the call synchronises
 * the stream once to read the out-of-range flag). */
atf_status atf_space_decode_indices128(const atf_space* s, const uint64_t* d_idx_lo, const uint64_t* d_idx_hi,
                                       int64_t n, int32_t* d_out, int64_t ld, void* stream);
atf_status atf_space_decode_range(const atf_space* s, uint64_t first_lo, uint64_t first_hi, int64_t n, int32_t* d_out,
                                  int64_t ld, void* stream);

/* int64 configurations (P:57 values of any integer type; reading #22): the same decoders with
 * int64 SoA output (column p at d_out + p*ld), valid on every generated space (an int32
 * space's values are sign-extended).  Rows out of range are filled with INT64_MIN and the call
 * returns ATF_ERR_INDEX (after a stream sync); otherwise asynchronous on `stream`. */
atf_status atf_space_decode_indices_i64(const atf_space* s, const uint64_t* d_idx, int64_t n, int64_t* d_out,
                                        int64_t ld, void* stream);
atf_status atf_space_decode_digits_i64(const atf_space* s, const uint64_t* d_digits, int64_t n, int64_t* d_out,
                                       int64_t ld, void* stream);
atf_status atf_space_decode_range_i64(const atf_space* s, uint64_t first_lo, uint64_t first_hi, int64_t n,
                                      int64_t* d_out, int64_t ld, void* stream);
/* 32 if every parameter value fits int32 (the int32 decoders, encode, neighbours and the
 * full-product filter apply), else 64.  Callable from BUILDING on. */
atf_status atf_space_value_bits(const atf_space* s, int32_t* bits);

/* Encode = inverse of decode (the index access of P:229-231 read
 * backwards, which also answers membership): d_values is a batch of n configurations,
 * int32 SoA (value of parameter p at d_values + p*ld, ld >= n).  Each row is located by a
 * top-down walk of every group's tree.  d_digits ([G][n] uint64, device) receives the
 * per-group leaf indices; a group whose values are not a valid prefix path gets
 * UINT64_MAX (the row is not in the space: not an error).  encode_indices also writes the
 * mixed-radix index d_idx[n] (group 0 most significant; UINT64_MAX for rows not in the
 * space) and needs S < 2^64 (else ATF_ERR_OVERFLOW).  Asynchronous on `stream`
 * (NULL = the space's stream); device buffers are borrowed until the work completes.
 * ATF_ERR_STATE before generate and on shard spaces; ATF_ERR_LIMIT on an int64 space. */
atf_status atf_space_encode_digits(const atf_space* s, const int32_t* d_values, int64_t n, int64_t ld,
                                   uint64_t* d_digits, void* stream);
atf_status atf_space_encode_indices(const atf_space* s, const int32_t* d_values, int64_t n, int64_t ld,
                                    uint64_t* d_digits, uint64_t* d_idx, void* stream);

/* CLTune-style baseline ("CLTune generates the search space
 * by filtering the full cartesian product"): every tuple of R_1 x ... x R_P is
 * enumerated on the GPU (no groups, no pruning of subtrees) and tested against the
 * constraints with the generic bytecode interpreter, parameter by parameter in declaration
 * order; a tuple is rejected at its first failing constraint, as a C++ conjunction of CLTune's
 * per-parameter std::function predicates would (the accepted set is the same).  *h_count =
 * the number of valid tuples (= S), *h_tuples (optional) = the product size.  Synchronous.
 * Needs only a planned space (callable before generate); ATF_ERR_OVERFLOW if the product is
 * >= 2^64; ATF_ERR_LIMIT on an int64 space. */
atf_status atf_space_filter_product(atf_space* s, uint64_t* h_count, uint64_t* h_tuples);

/* Random neighbours for simulated annealing ("a random neighbor c' of the
 * current configuration c"; SURVEY.md §8(f) NEXT-1 reading: c' = c with ONE parameter
 * re-drawn uniformly from its range such that c' is again a valid configuration).
 * d_in / d_out: n configurations, int32 SoA (ld_in / ld_out >= n; d_out may not alias
 * d_in).  Per row up to max_tries draws (counter-based splitmix64 of seed, row, draw);
 * the first draw whose row is in the space (tree walk of the changed parameter's group)
 * is kept.  d_moved[i] = the changed parameter id, or -1 (row copied unchanged).  Rows of
 * d_in must be valid configurations.  Asynchronous on `stream`.  ATF_ERR_STATE before
 * generate and on shard spaces; ATF_ERR_LIMIT on an int64 space. */
atf_status atf_space_neighbors(const atf_space* s, const int32_t* d_in, int64_t ld_in, int64_t n, uint64_t seed,
                               int32_t max_tries, int32_t* d_out, int64_t ld_out, int32_t* d_moved, void* stream);

/* Checkpoint / resume ("serialise spec + level arrays"): a generated space to a
 * file and back, so that a tuning run (decode / encode / neighbours) resumes without
 * regenerating.  atf_space_save writes the spec (names, int64 range values in range order,
 * constraint programs) and every group's level arrays (path records, CSR); synchronous.
 * ATF_ERR_STATE unless GENERATED by atf_space_generate (not a shard / rank part);
 * ATF_ERR_INVALID_ARG if the file cannot be written.
 * atf_space_load creates a space with `opts` (device, stream, allocator, flags), re-plans the
 * stored spec (groups and record layout must match the file), uploads the arrays and leaves it
 * GENERATED (size / decode / encode / neighbours / stats work; a later generate recomputes it).
 * A malformed, truncated or corrupted file (FNV-1a checksum) -> ATF_ERR_INVALID_ARG.  *out is
 * set even on error (atf_space_last_error explains; destroy it). */
atf_status atf_space_save(const atf_space* s, const char* path);
atf_status atf_space_load(const atf_space_opts* opts, const char* path, atf_space** out);

/* Per (group, level) statistics, in (group, level) order. */
typedef struct {
  int32_t group, level, param;
  int64_t r;        /* range size r_k                         */
  uint64_t evals;   /* candidate evaluations f_{k-1} * r_k    */
  uint64_t f;       /* nodes f_k                              */
  float ms;         /* device time of the level (ATF_FLAG_TIMING), else -1 */
  int32_t path;     /* 0 = fast atoms, 1 = generic interpreter */
  float expand_ms;  /* device time of the level's expand kernel alone (ATF_FLAG_TIMING), else -1 */
  int32_t kernel;   /* expand kernel: 0 = narrow (r <= 64), 1 = block-tile wide, 2 = warp-tile wide,
                       3 = narrow fast, 4 = narrow fast specialised at run time (NVRTC),
                       5 = fused narrow tail (tail_count + tail_emit, attributed to the tail's
                       first level; its other levels report 0 ms), 6 = the same specialised at
                       run time (NVRTC) */
  uint64_t pairs;   /* ATF_FLAG_TIMING: (node, candidate) pairs evaluated = evals, except on
                       warp-tile levels with a hot filter: the pairs the hot loop tested (the rest
                       are rejected by the per-segment |x| bounds: x | n needs |x| <= |n|, d | x
                       needs |x| >= |d|).  0 without ATF_FLAG_TIMING */
  int32_t cpt;      /* warp-tile levels: candidates per lane per segment (else 0)          */
  int32_t nseg;     /* warp-tile levels: candidate segments of 32 * cpt per node (else 0)  */
  int32_t launches; /* kernels the library launched for this level in the last generation
                       (expand + scan + emit, a re-run after an arena overflow included)    */
} atf_level_stats;
atf_status atf_space_stats(const atf_space* s, atf_level_stats* out, int32_t cap, int32_t* n_out);

/* Destroy (NULL ok).  Frees are stream-ordered on the space's stream. */
void atf_space_destroy(atf_space* s);

const char* atf_status_str(atf_status st);
const char* atf_space_last_error(const atf_space* s);

#ifdef __cplusplus
}
#endif
#endif /* ATFGEN_H */
