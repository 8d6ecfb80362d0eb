/*
 * include/olap.h — C-ABI of the B200-native OLAP hot path.
 *
 * Method: Malik, Riha, Shea, El-Ghazawi, "Task Scheduling for GPU Accelerated
 * Hybrid OLAP Systems with Multi-core Support and Text-to-Integer Translation",
 * IPDPS Workshops 2012 (text at /root/reference/PAPER.md, cited as PAPER.md:line).
 *
 * The library answers batches of OLAP queries against a dense MOLAP cube held in
 * B200 HBM.  A query is Eq. 1
 *       Q(C_1(f_1,t_1), ..., C_N(f_N,t_N))
 * restricted to one cube resolution (reading R14): one inclusive index range
 * [f_i, t_i] per dimension plus one aggregate op from "count, sum, average,
 * maximum etc." (MIN added per reading R4).  The answer aggregates
 * every cell of the sub-cube ("area of limited search", PAPER.md:109-112,
 * Fig. 2), whose volume is Eq. 3 (corrected to
 * V = prod_i (t_i - f_i + 1), reading R1).  Text predicates are first translated
 * to integer member ids through one dictionary per text column (§III-F,
 * PAPER.md:252-256).
 *
 * Conventions (all functions):
 *   - return an olap_status; out-parameters are written only on OLAP_OK;
 *     olap_last_error() gives a thread-local message for the last failure.
 *   - the caller owns every buffer it passes; the library copies what it keeps
 *     before returning (the *_device variants are asynchronous on `stream` and
 *     their buffers must stay live until that stream reaches the call).
 *   - handles are owned by the library and released by *_destroy (NULL-safe).
 *   - a handle is bound to the CUDA device it was created on; device pointers
 *     passed to *_device calls must live on that device.
 *   - a CUDA error maps to OLAP_E_CUDA (message names the call); bad arguments
 *     to OLAP_E_INVALID; a query outside the cube to OLAP_E_RANGE (host-buffer
 *     calls fail the whole batch and name the first bad query and dimension).
 *   - the library never falls back to the CPU: without a usable CUDA device
 *     every compute entry point returns OLAP_E_CUDA.
 */
#ifndef OLAP_H_
#define OLAP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct olap_cube olap_cube; /* opaque: a dense cube, one shard of it, or a group of shards */
typedef struct olap_dict olap_dict; /* opaque: one text column's dictionary, immutable */

typedef enum {
    OLAP_OK = 0,
    OLAP_E_INVALID = -1,     /* bad argument (NULL, ndims, dtype, op, sizes) */
    OLAP_E_RANGE = -2,       /* a query range lies outside the cube */
    OLAP_E_NOMEM = -3,       /* device or host allocation failed */
    OLAP_E_CUDA = -4,        /* CUDA runtime error / no device */
    OLAP_E_NCCL = -5,        /* NCCL missing, a NCCL call failed, or a communicator failed (asynchronously) */
    OLAP_E_STATE = -6,       /* handle in the wrong state */
    OLAP_E_UNSUPPORTED = -7
} olap_status;

typedef enum { OLAP_INT32 = 1, OLAP_FLOAT32 = 2 } olap_dtype; /* cell type, E_size = 4 B (Eq. 3) */

typedef enum { OLAP_SUM = 0, OLAP_COUNT = 1, OLAP_MIN = 2, OLAP_MAX = 3, OLAP_AVG = 4 } olap_agg;

typedef enum { OLAP_GEN_UNIFORM = 1, OLAP_GEN_AFFINE = 2 } olap_generator;

#define OLAP_RESULT_EMPTY 1u   /* some f_i > t_i: the box is empty (COUNT 0, SUM 0)        */
#define OLAP_RESULT_INVALID 2u /* *_device calls only: range out of bounds or bad op code    */

/* One condition C_i(f_i, t_i) of Eq. 1: inclusive index range; lo > hi => empty box. */
typedef struct { int64_t lo, hi; } olap_range;

/* One answer.  int32 cube: i = SUM, COUNT, MIN, MAX (exact; SUM is int64 with
 * two's-complement wraparound, reading R7), d = AVG.  float32 cube: d = SUM
 * (fp64 accumulation), MIN, MAX, AVG; i = COUNT.  AVG = (double)SUM/(double)V.
 * Fields not named for an op are 0. */
typedef struct { int64_t i; double d; uint32_t flags; uint32_t _pad; } olap_result;

/* Block-cyclic sharding of dimension 0 (reading R3 / DESIGN.md "layout"): global
 * row r belongs to shard (r / block) % nshards and is stored at local row
 * (r / (block*nshards))*block + r % block.  {1, 0, 1} (or NULL) = whole cube. */
typedef struct { int64_t nshards, shard, block; } olap_shard;

/* Per-query partial aggregates of one shard, structure-of-arrays in device
 * memory, combinable across shards with two element-wise reductions:
 *   sum[q]        int64: int32 cube -> wraparound sum (combine: +),
 *                         float32 cube -> the bits of a double (combine: + as float64)
 *   ext[2q+0]     int32: order-preserving code of the shard's MAX  (combine: max)
 *   ext[2q+1]     int32: bitwise NOT of the code of its MIN        (combine: max)
 * Identity (shard holds no cell of the box): sum 0, ext INT32_MIN.  The code of
 * an int32 cell is the cell; of a float32 cell, its bits b ^ ((b >> 31) & 0x7fffffff). */

/* ---------------------------------------------------------------- cube */

/* Create an uninitialised cube (or one shard of it) of ndims in [1,8] with the
 * given global extents (each >= 1), cell dtype, on CUDA `device`.  Layout:
 * row-major, dimension 0 outermost (PAPER.md:111-112 leaves the structure open;
 * reading R3).  OLAP_E_NOMEM if the shard does not fit in HBM. */
int olap_cube_create(int ndims, const int64_t* extents, int dtype, const olap_shard* shard,
                     int device, olap_cube** out);

/* Cell layouts in HBM.  The API is layout-blind: ranges, load, fill
 * and results always use the logical row-major index of Eq. 1's coordinates. */
#define OLAP_LAYOUT_ROWMAJOR 0 /* row-major, dim 0 outermost (olap_cube_create) */
#define OLAP_LAYOUT_BRICK 1    /* the last two dims stored in 4 x 8-cell bricks */
#define OLAP_LAYOUT_BRICK3 2   /* the last three dims stored in 2 x 4 x 4-cell bricks */

/* olap_cube_create with a layout.  OLAP_LAYOUT_BRICK (the "array chunking" of related
 * work [13], applied to the two innermost dimensions; reading R26): cells
 * (x_{N-2}, x_{N-1}) are grouped into bricks of 4 x 8 cells = 128 B, one B200 DRAM fetch
 * line, stored row-major inside the brick and in brick order (dims 0..N-3, brick row,
 * brick column).  A small box then costs ~half the DRAM lines it costs row-major (C5).
 * Needs ndims in [3,6] (dim 0 stays unbricked, so olap_shard is unchanged); extents
 * need not be multiples of 4 / 8 (padding cells are zero and never read).  Roll-up,
 * cube sets and olap_cube_add_facts_device return OLAP_E_UNSUPPORTED on such a cube;
 * olap_cube_info reports the padded brick storage.
 * OLAP_LAYOUT_BRICK3: the same over the three innermost dimensions, bricks of 2 x 4 x 4 cells
 * (x_{N-3}, x_{N-2}, x_{N-1}; still 128 B).  Small boxes of 3-D cubes whose cells spread over
 * all three dimensions (C5) touch ~11% fewer DRAM lines than with 4 x 8 bricks
 * (profiles/model_r02_c5_bricks.txt).  When ndims = 3 the pairs are of SHARD-LOCAL dim-0 rows
 * (block-cyclic ownership is unchanged: a query's owned rows are one local range).
 * Other layouts: OLAP_E_INVALID. */
int olap_cube_create_layout(int ndims, const int64_t* extents, int dtype, const olap_shard* shard,
                            int device, int layout, olap_cube** out);

/* Local geometry: owned dim-0 rows, owned cells, device pointer of the cells. */
int olap_cube_info(const olap_cube* c, int64_t* local_rows, int64_t* local_cells, void** d_cells);

/* Copy cells from a HOST array holding the FULL global cube in row-major order
 * (ncells must equal the product of the extents); a shard copies its own rows. */
int olap_cube_load(olap_cube* c, const void* cells, int64_t ncells);

/* Copy global dim-0 rows [row_lo, row_hi) from a HOST buffer holding exactly
 * those rows (row-major); rows not owned by this shard are skipped. */
int olap_cube_load_rows(olap_cube* c, int64_t row_lo, int64_t row_hi, const void* cells);

/* Fill on the device with a counter-based generator of the GLOBAL linear index i:
 *   OLAP_GEN_UNIFORM: z = splitmix64(seed, i); int32 -> (z >> 43) - 2^20,
 *                     float32 -> (z >> 40) * 2^-24
 *   OLAP_GEN_AFFINE:  v(x) = params[0] + sum_d params[1+d] * x_d  (ndims+1 params). */
int olap_cube_fill(olap_cube* c, int generator, uint64_t seed, const double* params);

int olap_cube_destroy(olap_cube* c);

/* Build step ("the GPU performs ... building the cube from relational
 * tables stored in GPU memory"): add nrows fact rows into the cells they
 * map to.  d_ids[d*nrows + r] is row r's member id in dimension d (DEVICE, int32, inside
 * [0, n_d)); d_values (DEVICE, nrows cells of the cube's dtype) or NULL to add 1 per
 * row (a fact-count cube).  Rows whose dim-0 id is not owned by this shard are skipped.
 * Cells are NOT cleared first (olap_cube_fill with params {0,...} or load zeros).
 * int32 adds are exact (wraparound, atomic, order-free).  float32 adds are deterministic:
 * the rows are sorted by cell (stable radix sort), each cell's values are added in row
 * order in fp64 and the cell becomes (float)((double)cell + sum), rounded once -- bit-equal
 * to oracle_factbuild.  float32 calls take < 2^31 rows and stream-ordered scratch of ~24 B
 * per row.  Asynchronous on `stream`. */
int olap_cube_add_facts_device(olap_cube* c, int64_t nrows, const int32_t* d_ids, const void* d_values,
                               void* stream);

/* ---------------------------------------------------------------- queries */

/* Whole path on HOST buffers: validate, copy ranges (nq*ndims, query-major) and
 * ops in, plan + range-reduce + finalize on the GPU, copy results out, sync.
 * Valid on an unsharded cube, on a group handle (olap_cube_create_multi: every shard
 * reduces, the partials are exchanged over NCCL, devices[0] finalizes) and on a shard with
 * an attached communicator (olap_cube_attach_comm: a collective, every rank passes the same
 * batch and receives every answer).  A plain shard returns OLAP_E_STATE.  nq == 0 is a no-op. */
int olap_query_batch(olap_cube* c, int64_t nq, const olap_range* ranges, const int32_t* ops,
                     olap_result* results);

/* Same path on DEVICE buffers, asynchronous on `stream` (cudaStream_t, NULL =
 * legacy default stream).  Invalid queries are flagged OLAP_RESULT_INVALID in
 * their result instead of failing the batch.  On a group handle the buffers and `stream`
 * live on devices[0] (the inputs are copied to the other devices over NVLink); on a shard
 * with a communicator, on its device (a collective, as above).  An unsharded cube's call can be
 * captured into a CUDA graph (and olap_query_partials_device likewise) after one
 * uncaptured call with at least nq queries has sized the cube's workspace; a replayed
 * graph must not overlap another batch on the same cube. */
int olap_query_batch_device(olap_cube* c, int64_t nq, const olap_range* d_ranges,
                            const int32_t* d_ops, olap_result* d_results, void* stream);

/* Shard-local half of the path: plan + range-reduce of this shard's part of
 * every query into partials (d_sum[nq], d_ext[2*nq], see above).  COUNT queries
 * and boxes that miss the shard produce the identity.  Asynchronous.  Not on a group
 * handle (OLAP_E_UNSUPPORTED: call it on the shards). */
int olap_query_partials_device(olap_cube* c, int64_t nq, const olap_range* d_ranges,
                               const int32_t* d_ops, int64_t* d_sum, int32_t* d_ext, void* stream);

/* Fold partials `in` into `acc` element-wise (the exchange's reduction, for
 * shards that live on one device).  Asynchronous. */
int olap_partials_combine_device(int dtype, int64_t nq, const int64_t* d_sum_in,
                                 const int32_t* d_ext_in, int64_t* d_sum_acc, int32_t* d_ext_acc,
                                 void* stream);

/* Turn fully-combined partials into results: COUNT = V (global volume, Eq. 3),
 * AVG = SUM/V, EMPTY / INVALID flags.  `extents` is a HOST array of the global
 * extents.  Asynchronous. */
int olap_finalize_device(int ndims, const int64_t* extents, int dtype, int64_t nq,
                         const olap_range* d_ranges, const int32_t* d_ops, const int64_t* d_sum,
                         const int32_t* d_ext, olap_result* d_results, void* stream);

/* Host-only helper (no GPU needed): the local dim-0 range [*llo, *lhi] of global
 * rows [lo, hi] on a shard of a dimension of n0 rows; *llo > *lhi if none. */
int olap_shard_local_rows(int64_t n0, const olap_shard* shard, int64_t lo, int64_t hi,
                          int64_t* llo, int64_t* lhi);

/* Accumulated device time (CUDA events on the launching stream) and launch
 * count of the range-reduce kernel since the last reset, plus the algorithmic
 * bytes it read (sum over non-COUNT queries of V_local * 4, Eq. 3).  Timing is
 * recorded only while enabled; enabling resets the counters. */
int olap_cube_profile(olap_cube* c, int enable);
int olap_cube_profile_read(olap_cube* c, double* reduce_ms, int64_t* launches, int64_t* bytes);

/* Kernels this cube has launched so far (plan, order, reduce; fill and fact build
 * included) and whether the L2-aware item order is active (cubes > 64 MiB). */
int olap_cube_stats(const olap_cube* c, int64_t* kernel_launches, int* l2_order);

/* Number of finalize kernels launched by this process (not bound to a cube). */
int64_t olap_finalize_launches(void);

/* Tile-shared scan: cubes larger than 64 MiB may answer a batch by staging
 * each 64-KiB tile of the cube into shared memory once and reducing every (query, tile)
 * pair from there, instead of streaming each query's own bytes from L2/HBM.  The device
 * picks the path per batch from the batch's reuse; results are identical in kind (bit-exact
 * for int32, within the float tolerance otherwise).  enabled = the cube has the tile path;
 * tile_cells = cells of a full tile; ntiles = tiles of the (local) cube; last_used = the
 * last batch took it (waits for that batch).  Any out-pointer may be NULL. */
int olap_cube_tile_stats(olap_cube* c, int* enabled, int64_t* tile_cells, int64_t* ntiles, int* last_used);

/* ---------------------------------------------------------------- multi-GPU */

/* The cube sharded on dimension 0 over several GPUs (BASELINE.json north_star part (4); the
 * paper used one GPU).  Every shard reduces its part of each query into the
 * partials above; ONE exchange combines them (16 B per query: sum with +, the two codes with
 * max, in one ncclGroup); the finalize turns them into answers.  Two ways to run it:
 *   - one process, several GPUs: olap_cube_create_multi -> a group handle.  The shards'
 *     partials are reduced over NCCL (ncclCommInitAll, ncclReduce) to devices[0];
 *   - one process per GPU: olap_comm_init_rank on every rank (the id from olap_comm_unique_id
 *     on rank 0, passed out of band), olap_cube_create with olap_shard {nranks, rank, b},
 *     then olap_cube_attach_comm.  ncclAllReduce: every rank gets every answer.
 * NCCL is loaded at run time (libnccl.so.2, or the file named by $OLAP_NCCL_LIB); without it
 * these calls return OLAP_E_NCCL.  After each exchange the communicators' asynchronous error
 * state is polled; a failed communicator is aborted and every later batch returns OLAP_E_NCCL.
 * Float sums are combined in NCCL's fixed order for a given configuration (deterministic);
 * int32 results are bit-exact for any number of shards (wraparound sums, R7). */

typedef struct {
    int32_t ndevices;          /* >= 1 distinct CUDA ordinals in `devices`; devices[0] is the root */
    int32_t shards_per_device; /* >= 1: G = ndevices * shards_per_device shards, shard g on devices[g / spd];
                                  shards of one device are folded in shard order before the exchange */
    const int32_t* devices;
    int64_t shard_block;       /* block-cyclic dim-0 block b >= 1 (olap_shard) */
    int32_t layout;            /* OLAP_LAYOUT_* of every shard */
    int32_t _pad;
} olap_cube_opts;

/* A group handle: G shard cubes (olap_shard {G, g, shard_block}) over opts->devices.  load,
 * load_rows, fill, destroy, info (summed rows / cells, d_cells = NULL), profile, stats and the
 * query calls act on every shard.  OLAP_E_NCCL if NCCL cannot be loaded or initialised. */
int olap_cube_create_multi(int ndims, const int64_t* extents, int dtype, const olap_cube_opts* opts,
                           olap_cube** out);

typedef struct olap_comm olap_comm;               /* opaque: one rank of a NCCL communicator */
typedef struct { char internal[128]; } olap_comm_id;  /* = ncclUniqueId */

/* Rank 0 creates the id and broadcasts its 128 bytes to every rank (any channel). */
int olap_comm_unique_id(olap_comm_id* id);
/* Collective over nranks processes: this rank's communicator on CUDA `device`. */
int olap_comm_init_rank(const olap_comm_id* id, int nranks, int rank, int device, olap_comm** out);
int olap_comm_info(const olap_comm* comm, int* nranks, int* rank, int* device);
/* Poll the asynchronous error state (OLAP_E_NCCL, and the communicator is aborted, on failure). */
int olap_comm_check(olap_comm* comm);
/* Destroys (or aborts, after a failure) the communicator; detach it from cubes first. */
int olap_comm_destroy(olap_comm* comm);

/* Attach (comm != NULL) or detach a communicator to a shard whose olap_shard is {nranks, rank,
 * b} on the communicator's device: olap_query_batch(_device) and olap_query_stream then run the
 * whole sharded path as a collective.  The cube borrows the communicator. */
int olap_cube_attach_comm(olap_cube* c, olap_comm* comm);

/* The exchange alone (all-reduce in place of d_sum[nq], d_ext[2*nq] over the communicator),
 * asynchronous on `stream`, for callers that run olap_query_partials_device themselves. */
int olap_exchange_partials_device(olap_comm* comm, int dtype, int64_t nq, int64_t* d_sum, int32_t* d_ext,
                                  void* stream);
int olap_nccl_version(int* version);

/* A stream of nq queries (HOST buffers) answered in batches of `batch` (<= 0: one batch),
 * pipelined: batch k+1's copy-in and range-reduce run while batch k's exchange, finalize and
 * copy-out complete ("overlap batch k's exchange with batch k+1's reduction").
 * Any cube kind (plain, group, shard with a communicator).  Results are those of
 * olap_query_batch on each batch; the whole stream fails with OLAP_E_RANGE on a bad query. */
int olap_query_stream(olap_cube* c, int64_t nq, const olap_range* ranges, const int32_t* ops,
                      olap_result* results, int64_t batch);

/* ---------------------------------------------------------------- dictionaries */

/* Build one text column's dictionary from n keys (key i = bytes[offsets[i],
 * offsets[i+1]), HOST buffers, length-delimited, NUL not special, duplicates
 * allowed).  Ids are the ranks of the distinct keys in byte-lexicographic
 * (memcmp, shorter-prefix-first) order (reading R11).  The sorted arena and an
 * open-addressing hash table are uploaded to `device`. */
int olap_dict_build(const char* bytes, const int64_t* offsets, int64_t n, int device,
                    olap_dict** out);

int olap_dict_size(const olap_dict* d, int64_t* n_distinct);

/* Translate n keys (HOST buffers) to ids on the GPU, key i looked up in
 * dicts[dict_of_key[i]] (dict_of_key NULL => dicts[0]); ids_out[i] = -1 when
 * absent (reading R13).  *n_missing (optional) = number of misses.  All dicts
 * must live on one device. */
int olap_dict_translate(const olap_dict* const* dicts, int ndicts, const int32_t* dict_of_key,
                        const char* bytes, const int64_t* offsets, int64_t n, int32_t* ids_out,
                        int64_t* n_missing);

/* Same on DEVICE buffers (bytes, offsets[n+1], dict_of_key or NULL, ids_out),
 * asynchronous on `stream`; d_n_missing (device int64, optional) is incremented. */
int olap_dict_translate_device(const olap_dict* const* dicts, int ndicts,
                               const int32_t* d_dict_of_key, const char* d_bytes,
                               const int64_t* d_offsets, int64_t n, int32_t* d_ids_out,
                               int64_t* d_n_missing, void* stream);

/* For string-range conditions: out[i] = number of members < key i (upper = 0,
 * lower_bound) or <= key i (upper = 1, upper_bound), by binary search on the
 * GPU; HOST buffers.  A range [s1, s2] maps to ids [lower(s1), upper(s2) - 1]. */
int olap_dict_bound(const olap_dict* d, const char* bytes, const int64_t* offsets, int64_t n,
                    int upper, int32_t* out);

/* Text conditions -> Eq. 1 ranges (PAPER.md:252-256 with readings R11/R13).  One
 * condition per (query, dimension), kinds[q*ndims + d]:
 *   OLAP_COND_ALL    whole dimension [0, n_d - 1]; consumes no key
 *   OLAP_COND_EQ     one key s: [id, id] with id = dicts[d][s]; a missing key gives an
 *                    empty box [1, 0] and is counted in *n_missing
 *   OLAP_COND_RANGE  two keys s1, s2: [lower_bound(s1), upper_bound(s2) - 1] (ids are
 *                    sorted ranks, so this is every member with s1 <= member <= s2;
 *                    empty when no member lies in between)
 *   OLAP_COND_IDS    numeric condition: ranges_in[q*ndims + d] copied as given
 * Keys are consumed in (q, d) order from bytes/offsets (nkeys keys).  dicts[d] may
 * be NULL for a dimension that only uses ALL/IDS; a text dimension's extent must be
 * its dictionary's size.  HOST buffers; translation runs on the dictionaries' GPU. */
typedef enum { OLAP_COND_ALL = 0, OLAP_COND_EQ = 1, OLAP_COND_RANGE = 2, OLAP_COND_IDS = 3 } olap_cond_kind;

int olap_text_ranges(const olap_dict* const* dicts, int ndims, const int64_t* extents, int64_t nq,
                     const int32_t* kinds, const olap_range* ranges_in, const char* bytes,
                     const int64_t* offsets, int64_t nkeys, olap_range* ranges_out, int64_t* n_missing);

/* Same on DEVICE buffers, asynchronous on `stream`: d_first_key[q*ndims + d] is the
 * index of the condition's first key (any value for ALL/IDS); d_ranges_in may be NULL
 * when no IDS condition is present; d_n_missing (device int64, optional) is incremented.
 * `extents` is a HOST array. */
int olap_text_ranges_device(const olap_dict* const* dicts, int ndims, const int64_t* extents, int64_t nq,
                            const int32_t* d_kinds, const int64_t* d_first_key,
                            const olap_range* d_ranges_in, const char* d_bytes, const int64_t* d_offsets,
                            int64_t nkeys, olap_range* d_ranges_out, int64_t* d_n_missing, void* stream);

/* Inverse: bytes of member `id` (pointer valid until the dict is destroyed). */
int olap_dict_lookup(const olap_dict* d, int32_t id, const char** bytes, int64_t* len);

int olap_dict_destroy(olap_dict* d);

/* ---------------------------------------------------------------- fact tables */

/* The paper's GPU data structure (§III-E): a fact
 * table of nrows rows held in GPU memory as one 1-D array of columns "one after
 * another".  Dimension columns hold int32 member ids (one column per dimension x
 * level, e.g. translated text); data columns hold int32 or float32
 * measures.  At most 16 columns. */
typedef struct olap_table olap_table;

/* One condition C_L(f, t, l_K) of a query Q_D (Eq. 11): column `col`
 * (an int32 dimension column) and an inclusive id range [lo, hi]; lo > hi matches
 * nothing. */
typedef struct { int32_t col; int32_t _pad; int64_t lo, hi; } olap_cond;

int olap_table_create(int64_t nrows, int ncols, const int32_t* col_dtypes, int device, olap_table** out);

/* Copy column `col` (nrows 4-byte values, HOST buffer). */
int olap_table_load_column(olap_table* t, int col, const void* values);

/* Device pointer of column `col` (nrows 4-byte values), e.g. to fill it on the device. */
int olap_table_column_device(olap_table* t, int col, void** d_ptr);

/* A table's calls (and a partition's) may come from different streams: each workspace orders
 * a batch after the previous batch on that workspace (an event), whatever its stream.
 * Answer nq queries Q_D on HOST buffers.  Query q has conditions
 * conds[cond_offsets[q] .. cond_offsets[q+1]) (at most 16; cond_offsets[0] = 0), data
 * column data_cols[q] and op ops[q].  A row matches when it satisfies every condition
 * (PAPER.md:208); the result aggregates the data column over matching rows: COUNT =
 * matching rows (facts), SUM (int64 wraparound / fp64), MIN, MAX, AVG = SUM / COUNT.
 * No matching row: OLAP_RESULT_EMPTY.  One shared scan answers the whole batch. */
int olap_table_query_batch(olap_table* t, int64_t nq, const int64_t* cond_offsets, const olap_cond* conds,
                           const int32_t* data_cols, const int32_t* ops, olap_result* results);

/* Same on DEVICE buffers, asynchronous on `stream`; malformed queries are flagged
 * OLAP_RESULT_INVALID. */
int olap_table_query_batch_device(olap_table* t, int64_t nq, const int64_t* d_cond_offsets,
                                  const olap_cond* d_conds, const int32_t* d_data_cols, const int32_t* d_ops,
                                  olap_result* d_results, void* stream);

/* Accumulated device time (CUDA events on the launching stream) and launch count of the scan
 * kernel of the table's own calls (not its partitions') since profiling was enabled; enabling
 * resets the counters. */
int olap_table_profile(olap_table* t, int enable);
int olap_table_profile_read(olap_table* t, double* scan_ms, int64_t* launches);

int olap_table_destroy(olap_table* t);

/* A GPU partition for fact-table queries (Fig. 7: the paper
 * splits its C2070 into partitions of 1, 2 and 4 SMs so several queries are answered
 * concurrently, each by one partition).  A partition launches the scan on at most
 * sm_count SMs' worth of blocks (sm_count x resident blocks per SM; sm_count <= 0 or
 * above the device's SM count = every SM) with its own workspace, so partitions of one
 * table may run concurrently on different streams.  Every scan reads only the columns
 * the batch references: its conditions' columns plus, unless every query is COUNT,
 * their data columns (Eq. 12). */
typedef struct olap_table_part olap_table_part;
int olap_table_part_create(olap_table* t, int sm_count, olap_table_part** out);
int olap_table_part_sms(const olap_table_part* p, int* sm_count, int* blocks);

/* olap_table_query_batch_device on the partition. */
int olap_table_part_query_device(olap_table_part* p, int64_t nq, const int64_t* d_cond_offsets,
                                 const olap_cond* d_conds, const int32_t* d_data_cols, const int32_t* d_ops,
                                 olap_result* d_results, void* stream);

/* Queries given as boxes over dimension columns, e.g. olap_text_ranges output: query q's
 * condition on dimension d is column dim_cols[d] in d_boxes[q*ndims + d] (inclusive); a
 * range covering all of [0, extents[d]) is no condition and reads no column (Eq. 12); an
 * empty range (lo > hi) matches nothing; lo < 0 or hi >= extents[d] flags the query
 * OLAP_RESULT_INVALID (the cube path's rule, reading R10).  dim_cols and extents are HOST arrays of ndims <= 16. */
int olap_table_part_query_boxes_device(olap_table_part* p, int64_t nq, int ndims, const int32_t* dim_cols,
                                       const int64_t* extents, const olap_range* d_boxes,
                                       const int32_t* d_data_cols, const int32_t* d_ops, olap_result* d_results,
                                       void* stream);
int olap_table_part_destroy(olap_table_part* p);

/* ---------------------------------------------------------------- dispatcher (NEXT #4) */

/* The paper's scheduling algorithm, Fig. 10 (§III-G), host code.
 * Every query Q gets a deadline T_D = T_O + T_C.  Fig. 10 estimates Q's response time on
 * every partition, then picks one:
 *   - a cube partition that meets T_D and beats the fastest table partition;
 *   - otherwise the slowest table partition that meets T_D;
 *   - otherwise the partition that answers first.
 * The partition's queue time T_Q is then advanced.  olap_sched_complete applies the
 * paper's correction: real minus estimated processing time is added to
 * the queue's T_Q.
 *
 * Performance function of a partition, Eq. 4, generalised:
 *     T(x) = a1 * x^p1 + b1   if x < x_split        (range A)
 *            a2 * x^p2 + b2   otherwise             (range B, reading R25)
 * Eq. 7 / Eq. 10 (CPU cube model, x = SC_size in MB) and Eq. 14-15 (GPU table model,
 * x = C_QD / C_TOTAL) are instances, and so is the B200 roofline T = bytes / BW + t0
 * (DESIGN.md §8(f)). */
typedef struct { double x_split, a1, p1, b1, a2, p2, b2; } olap_perf_fn;
typedef enum { OLAP_PART_CUBE = 0, OLAP_PART_TABLE = 1 } olap_part_kind;
/* CUBE partitions play the paper's CPU OLAP partition (answers from pre-computed cubes,
 * x = cube_mb), TABLE partitions its GPU partitions (fact-table scan, x = col_frac).
 * Partitions are listed in the order Fig. 10's FOR loop visits them (slow -> fast).
 * needs_translation: the partition's queries pass through the translation queue first
 * (the paper: GPU partitions only). */
typedef struct { int32_t kind; int32_t needs_translation; olap_perf_fn perf; } olap_sched_partition;
/* t_arrival = T_O (s); cube_mb = SC_size (Eq. 3) in MB of the cube that answers Q, < 0 if
 * none can; col_frac = C_QD / C_TOTAL (Eq. 12-13), < 0 if no table can; t_trans = T_TRANS
 * (Eq. 18) in s, 0 when Q has no text parameter. */
typedef struct { double t_arrival, cube_mb, col_frac, t_trans; } olap_sched_query;
/* partition = chosen index (-1: no partition can answer Q); translated = Q goes through the
 * translation queue; t_response = estimated T_R; t_deadline = T_D; t_est = estimated
 * processing time on the chosen partition (pass it back to olap_sched_complete). */
typedef struct { int32_t partition, translated; double t_response, t_deadline, t_est; } olap_sched_decision;
typedef struct olap_sched olap_sched;

/* nparts in [1, 64]; t_c = T_C > 0 (s), +inf allowed. */
int olap_sched_create(int nparts, const olap_sched_partition* parts, double t_c, olap_sched** out);
/* Schedule n queries in order (online: each sees the queue state the previous left). */
int olap_sched_submit(olap_sched* s, int64_t n, const olap_sched_query* qs, olap_sched_decision* out);
int olap_sched_complete(olap_sched* s, int partition, double t_est, double t_real);
/* t_q[0..nparts-1] = T_Q of every partition, t_q[nparts] = T_Q|TRANS. */
int olap_sched_queues(const olap_sched* s, double* t_q);
int olap_sched_destroy(olap_sched* s);

/* ---------------------------------------------------------------- multi-resolution cube set */

/* Resolution hierarchy (Fig. 1: "years (low resolution), months, days,
 * hours (high resolution)"): levels 0 (coarsest) .. nlevels-1 (finest) for every
 * dimension.  level_ids[d*nlevels + r] points to n_finest[d] int32: the level-r member of
 * each finest member of dimension d; ids start at 0 and step by 0 or 1 (every coarse
 * member is a contiguous block), the finest level is the identity, and a member never
 * splits a member of a coarser level.  A dimension without a hierarchy passes the
 * identity at every level.  HOST buffers, copied. */
typedef struct olap_hier olap_hier;
int olap_hier_create(int ndims, int nlevels, const int64_t* n_finest, const int32_t* const* level_ids,
                     olap_hier** out);
int olap_hier_extents(const olap_hier* h, int level, int64_t* extents /* ndims */);

/* Conditions of Eq. 1 given at their own resolution r (levels[q*ndims + d]) expressed at
 * level `target` >= r: [f, t] -> [first target member in f, last target member in t].
 * Empty stays empty; out of bounds -> OLAP_E_RANGE.  HOST buffers. */
int olap_hier_convert(const olap_hier* h, int64_t nq, const olap_range* ranges, const int32_t* levels,
                      int target, olap_range* out);

/* Pre-calculate a coarser cube: coarse cell = SUM (or MIN / MAX) of the
 * fine cells mapping to it, computed on the GPU (int32 SUM wraps into int32 cells,
 * float32 SUM accumulates in fp64 and rounds once).  Both cubes unsharded, on one device,
 * with extents equal to their levels' member counts.  Synchronous. */
int olap_cube_rollup(const olap_hier* h, const olap_cube* fine, int fine_level, olap_cube* coarse,
                     int coarse_level, int op);
int olap_hier_destroy(olap_hier* h);

/* A set of cubes at different resolutions sharing one hierarchy (cubes are borrowed,
 * not owned).  olap_cubeset_query routes every query by Eq. 2:
 * R = max_i r_i; the cube of resolution R answers it, its conditions converted to level
 * R.  SUM, which roll-up preserves, may also use the lowest-resolution finer cube.  A
 * query no cube can answer gets OLAP_RESULT_INVALID (answer it from the fact table,
 * olap_table_*, as the paper does on the GPU).  level_used[q] (optional) = cube level,
 * or -1.  HOST buffers. */
typedef struct olap_cubeset olap_cubeset;
int olap_cubeset_create(const olap_hier* h, olap_cubeset** out);
int olap_cubeset_add(olap_cubeset* s, int level, olap_cube* c);
int olap_cubeset_query(olap_cubeset* s, int64_t nq, const olap_range* ranges, const int32_t* levels,
                       const int32_t* ops, olap_result* results, int32_t* level_used);
int olap_cubeset_destroy(olap_cubeset* s);

/* ---------------------------------------------------------------- misc */

const char* olap_last_error(void); /* thread-local; valid until the next olap_* call */
const char* olap_version(void);

#ifdef __cplusplus
}
#endif
#endif /* OLAP_H_ */
