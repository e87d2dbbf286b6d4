/*
 * astitch.h — C ABI of the B200-native AStitch stitched-subgraph engine.
 *
 * What it does.  A memory-intensive subgraph (element-wise ops, row / column
 * reductions and broadcasts; Sec. 2.1) is described with the
 * graph builder below, planned once for a runtime shape (the paper's
 * just-in-time compilation, Sec. 4) and then executed as ONE
 * stitched kernel on the caller's CUDA stream (Sec. 3.2.2-3.2.3).
 * The plan chooses, per op, one of the four stitching schemes of Table 1
 * (independent, local = registers, regional = shared memory /
 * intra-team, global = HBM + grid barrier) and an adaptive thread mapping
 * (task packing / splitting, Sec. 3.3; shape rule P:L270).
 *
 * Conventions (every entry point):
 *   - Returns an astitch_status; ASTITCH_OK == 0.  On error a thread-local
 *     message is available from astitch_last_error().  No C++ exception ever
 *     crosses this boundary.
 *   - Handles (graph, plan, comm) are opaque, allocated by the library and
 *     released by the matching *_destroy.  A plan copies what it needs from
 *     the graph: the graph may be destroyed right after astitch_plan().
 *   - Every DEVICE buffer (inputs, outputs, workspace) is caller-owned.  The
 *     library never allocates, frees or memsets device memory inside
 *     astitch_run / astitch_run_sharded.
 *   - Streams are passed as `void*` holding a cudaStream_t / CUstream (NULL =
 *     the legacy default stream).  All device work is asynchronous on it.
 *   - Layouts: FULL = [rows, cols] row-major contiguous; ROWVEC = [rows];
 *     COLVEC = [cols]; LENGTHS = int32 [ceil(rows / rows_per_segment)].
 *     Base pointers must be 16-byte aligned (else ASTITCH_ERR_INVALID_ARGUMENT).
 *     Inputs are passed in the order of astitch_graph_input / _lengths calls,
 *     outputs in astitch_graph_output order.
 */
#ifndef ASTITCH_H_
#define ASTITCH_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ASTITCH_ABI_VERSION 1

typedef enum {
  ASTITCH_OK = 0,
  ASTITCH_ERR_INVALID_ARGUMENT = 1, /* null / misaligned pointer, bad enum, bad index   */
  ASTITCH_ERR_INVALID_GRAPH = 2,    /* kind / dtype mismatch while building the graph  */
  ASTITCH_ERR_UNSUPPORTED = 3,      /* pattern outside the IR (e.g. reduce of a ROWVEC)*/
  ASTITCH_ERR_SHAPE = 4,            /* rows < 0, cols < 1, size overflow               */
  ASTITCH_ERR_RESOURCE = 5,         /* no single-kernel plan fits (STRICT flag)        */
  ASTITCH_ERR_CUDA = 6,             /* driver / NVRTC failure (detail in last_error)   */
  ASTITCH_ERR_NCCL = 7,             /* NCCL failure                                    */
  ASTITCH_ERR_INTERNAL = 8
} astitch_status;

typedef enum { ASTITCH_F32 = 0, ASTITCH_BF16 = 1, ASTITCH_F16 = 2, ASTITCH_I32 = 3 } astitch_dtype;

/* Tensor kinds: the shape class of a value of the subgraph. */
typedef enum {
  ASTITCH_FULL = 0,    /* [rows, cols]                                   */
  ASTITCH_ROWVEC = 1,  /* [rows]   (one value per row)                   */
  ASTITCH_COLVEC = 2,  /* [cols]   (one value per column)                */
  ASTITCH_SCALAR = 3,  /* constant                                       */
  ASTITCH_LENGTHS = 4, /* int32 valid lengths, one per row segment       */
  ASTITCH_SEGMENTS = 5 /* int32 [nseg][4] packed varlen segment table    */
} astitch_kind;

/* Element-wise unary ops.  Light vs heavy follows P:L101 (heavy: exp, log,
 * tanh, erf, sqrt, rsqrt, rcp, sigmoid, gelu*; also binary DIV / POW). */
typedef enum {
  ASTITCH_NEG = 0, ASTITCH_ABS, ASTITCH_EXP, ASTITCH_LOG, ASTITCH_TANH, ASTITCH_ERF,
  ASTITCH_SQRT, ASTITCH_RSQRT, ASTITCH_RCP, ASTITCH_SIGMOID,
  ASTITCH_GELU_TANH,      /* 0.5 x (1 + tanh(sqrt(2/pi)(x + 0.044715 x^3)))      */
  ASTITCH_GELU_ERF,       /* 0.5 x (1 + erf(x / sqrt 2))                          */
  ASTITCH_GELU_TANH_GRAD, /* d/dx GELU_TANH                                       */
  ASTITCH_UNOP_COUNT
} astitch_unop;

typedef enum {
  ASTITCH_ADD = 0, ASTITCH_SUB, ASTITCH_MUL, ASTITCH_DIV, ASTITCH_MAX, ASTITCH_MIN, ASTITCH_POW,
  ASTITCH_BINOP_COUNT
} astitch_binop;

typedef enum { ASTITCH_SUM = 0, ASTITCH_RMAX = 1 } astitch_redop;

/* ROW: reduce over the contiguous dimension ([R,C] -> [R]); broadcast [R] -> [R,C].
 * COL: reduce over rows ([R,C] -> [C]);                      broadcast [C] -> [R,C].
 * (row-reduce vs column-reduce: Sec. 2.1.) */
typedef enum { ASTITCH_AXIS_ROW = 0, ASTITCH_AXIS_COL = 1 } astitch_axis;

typedef struct astitch_graph_s* astitch_graph_t;
typedef struct astitch_plan_s* astitch_plan_t;
typedef struct astitch_comm_s* astitch_comm_t;
typedef int32_t astitch_value_t;

/* ---------------------------------------------------------------- errors */
const char* astitch_status_str(astitch_status s);
/* Detail of the last error on the calling thread ("" if none).  Valid until the
 * next astitch_* call on the same thread. */
const char* astitch_last_error(void);
int astitch_abi_version(void);

/* ---------------------------------------------------------------- graph builder
 * The IR of the subgraph (the paper's stitch op, Sec. 4.1).  Builder
 * calls validate immediately and return ASTITCH_ERR_INVALID_GRAPH on a kind or
 * dtype mismatch (binary ops need equal kinds or a SCALAR operand; reduce takes
 * a FULL value; broadcast ROW takes a ROWVEC, broadcast COL a COLVEC). */
astitch_status astitch_graph_create(astitch_graph_t* out);
astitch_status astitch_graph_destroy(astitch_graph_t g);
/* A tensor input of kind FULL / ROWVEC / COLVEC and storage dtype F32 / BF16 / F16
 * (or kind LENGTHS with dtype I32: a mask bound later by astitch_graph_set_mask). */
astitch_status astitch_graph_input(astitch_graph_t g, astitch_kind kind, astitch_dtype dtype,
                                   astitch_value_t* out);
/* A SCALAR constant (applied in fp32 on the device, fp64 in the oracle). */
astitch_status astitch_graph_const(astitch_graph_t g, double v, astitch_value_t* out);
/* Element-wise ops: same kind as the operand(s), applied per
 * element in fp32 on the device.  MAX / MIN propagate NaN (reading R12).
 * Integer POW exponents 0..8 are repeated multiplication (R11). */
astitch_status astitch_graph_unary(astitch_graph_t g, astitch_unop op, astitch_value_t a,
                                   astitch_value_t* out);
astitch_status astitch_graph_binary(astitch_graph_t g, astitch_binop op, astitch_value_t a,
                                    astitch_value_t b, astitch_value_t* out);
/* Row (FULL -> ROWVEC) or column (FULL -> COLVEC) reduction.  Sums
 * accumulate in fp32 with a fixed order (bitwise run-to-run deterministic,
 * R13); a sum that is broadcast back into an add / sub (a mean) keeps the
 * spread of its row / column (shifted or fp64 sums applied as hi + lo: R7b,
 * R7c).  RMAX propagates NaN (R12).  A column reduction ends the pass over
 * the rows: its consumers run after a grid barrier (global stitching) in the
 * same kernel. */
astitch_status astitch_graph_reduce(astitch_graph_t g, astitch_redop op, astitch_axis axis,
                                    astitch_value_t a, astitch_value_t* out);
astitch_status astitch_graph_broadcast(astitch_graph_t g, astitch_axis axis, astitch_value_t a,
                                       astitch_value_t* out);
/* Key-padding mask (irregular sequence lengths; BASELINE configs[2]).  Adds an
 * int32 LENGTHS input (next in input order) of ceil(rows / rows_per_segment)
 * entries.  Element (r, c) is valid iff c < lengths[r / rows_per_segment].
 * Invalid elements are excluded from reductions (identity 0 for SUM, -inf for
 * RMAX) and written as 0 in FULL outputs.  At most one mask per graph. */
astitch_status astitch_graph_lengths(astitch_graph_t g, int64_t rows_per_segment,
                                     astitch_value_t* out);
/* The same mask in two steps (SURVEY 8(b)'s form): `lengths` is an existing
 * input created by astitch_graph_input(g, ASTITCH_LENGTHS, ASTITCH_I32, &v);
 * this call binds it as the graph's key-padding mask with rows_per_segment.
 * Errors: ERR_INVALID_ARGUMENT (NULL g, bad value, rows_per_segment < 1),
 * ERR_INVALID_GRAPH (not a LENGTHS input, or the graph already has a mask /
 * segments).  astitch_plan fails with ERR_INVALID_GRAPH if a LENGTHS input
 * was never bound. */
astitch_status astitch_graph_set_mask(astitch_graph_t g, astitch_value_t lengths, int64_t rows_per_segment);
/* Packed variable-length rows ("varlen" layout: irregular shapes without
 * padding, Sec. 3.3 Challenge II).  Adds an
 * int32 SEGMENTS input (next in input order) of nseg entries of 4 int32
 *     { row_start, cols, pitch, offset8 }:
 * segment s owns global rows [row_start_s, row_start_{s+1}) (row_start_0 = 0,
 * increasing, row_start_nseg := plan rows); each of its rows has `cols_s`
 * elements (1 <= cols_s <= plan cols), stored in EVERY FULL tensor (input and
 * output) at element offset 8*offset8_s + (r - row_start_s) * pitch_s, with
 * pitch_s a multiple of 8 and >= cols_s.  FULL tensors therefore hold `elems`
 * elements (>= the last segment's end); ROWVEC tensors stay [rows], COLVEC
 * [cols] (column c of any segment reads entry c).  The plan's cols is the
 * maximum row length: the thread mapping is chosen for it and shorter rows
 * are handled like key-padding masks (chunks past cols_s are skipped), but
 * nothing past a row is read and only whole 16-byte chunks up to cols_s are
 * written (elements cols_s .. next 16-byte boundary are written as 0, inside
 * the pitch).  Row-wise subgraphs only: column reductions, masks, sharding and
 * FORCE_GLOBAL are ERR_UNSUPPORTED with segments.  The table must be valid
 * (see astitch_segments_layout); it is read on the device and not checked. */
astitch_status astitch_graph_segments(astitch_graph_t g, int32_t nseg, int64_t elems,
                                      astitch_value_t* out);
/* Host helper: the canonical segment table for nseg segments of seg_rows[s]
 * rows x seg_cols[s] columns, packed back to back in segment order with
 * pitch = cols rounded up to a multiple of 8 elements.  Writes table[4*nseg],
 * *rows = total rows and *elems = total elements per FULL tensor.
 * Errors: ERR_INVALID_ARGUMENT (NULL, nseg < 1, rows < 0, cols < 1),
 * ERR_SHAPE (offsets beyond 2^31 x 8 elements). */
astitch_status astitch_segments_layout(int32_t nseg, const int64_t* seg_rows, const int32_t* seg_cols,
                                       int32_t* table, int64_t* rows, int64_t* elems);
/* Marks value v as a stitch-op output stored with dtype (F32 / BF16 / F16).
 * FULL, ROWVEC and COLVEC values can be outputs. */
astitch_status astitch_graph_output(astitch_graph_t g, astitch_value_t v, astitch_dtype dtype,
                                    int32_t* out_index);

/* ---------------------------------------------------------------- planning */
enum {
  ASTITCH_FLAG_NO_COMPILE = 1u << 0,    /* plan + codegen only (host tests, no NVRTC)   */
  ASTITCH_FLAG_FORCE_GLOBAL = 1u << 1,  /* ablation: demote regional -> global (Table 4)*/
  ASTITCH_FLAG_NO_PACK = 1u << 2,       /* ablation: no horizontal packing (team = warp)*/
  ASTITCH_FLAG_NO_SPLIT = 1u << 3,      /* ablation: never split long rows             */
  ASTITCH_FLAG_STRICT_SINGLE_KERNEL = 1u << 4, /* ERR_RESOURCE if the planned one-wave grid is
                                           not co-resident (instead of shrinking it) */
  ASTITCH_FLAG_NO_TMA = 1u << 5,        /* do not use the TMA-staged packed template   */
  ASTITCH_FLAG_NO_PREFETCH = 1u << 6,   /* no software prefetch of the next row        */
  ASTITCH_FLAG_LAUNCH_CHECK = 1u << 7,  /* synchronise + check after every launch (debug)*/
  ASTITCH_FLAG_FORCE_SPLIT = 1u << 8,   /* ablation: split rows over clusters whenever the
                                           paper's shape rule holds (no B200 size threshold) */
  ASTITCH_FLAG_NO_PDL = 1u << 9,        /* launch without programmatic dependent launch   */
  ASTITCH_FLAG_DEBUG_BARRIER = 1u << 10 /* debug: a grid barrier waiting > 5 s prints and
                                           traps (a launch error) instead of spinning on */
};

typedef struct {
  int64_t rows;          /* rows of THIS process's shard (FULL / ROWVEC extent)        */
  int64_t cols;          /* >= 1                                                       */
  int32_t device;        /* CUDA ordinal; -1 = host-only plan (no module load, no run) */
  int32_t shard_rank;    /* 0 .. shard_world-1 (row partition index)                    */
  int32_t shard_world;   /* number of row shards (1 = unsharded)                        */
  uint32_t flags;        /* ASTITCH_FLAG_*                                              */
  int32_t sm_count;      /* 0 = query the device (host-only plans assume 148)           */
  int32_t reserved;
} astitch_plan_desc;

/* Plans graph g for desc: classify ops, find dominants and groups, choose the
 * thread mapping, propagate it, finalise the schemes, plan memory and the
 * launch configuration (Sec. 4.3-4.5); then generate the stitched
 * kernel and compile it for sm_100a with NVRTC (unless FLAG_NO_COMPILE) and
 * load it on desc.device (unless device == -1).
 * Errors: ERR_SHAPE (rows < 0, cols < 1, overflow), ERR_UNSUPPORTED,
 * ERR_RESOURCE (STRICT flag and the planned grid is not co-resident), ERR_CUDA
 * (NVRTC / load).  Every plan is ONE kernel: when a staged buffer would exceed
 * the shared memory of a block, the planner demotes the mapping (fewer
 * pipeline stages / tile rows / teams per block, or a register row team
 * instead of a staged tile: the paper's "until the memory usage is under the
 * limit"); describe()["demotions"] lists what it changed. */
astitch_status astitch_plan(astitch_graph_t g, const astitch_plan_desc* desc, astitch_plan_t* out);
/* astitch_plan with explicit overrides of the planner's choices, for
 * experiments and tests: `tuning` is NULL or "key=value,..." with integer
 * values; keys: threads, unroll, team, bps (fixed blocks/SM, no
 * assume-relax-apply), vec_bytes (16|32), hoist (0|1), tile_stages, tile_rows,
 * tile_threads, split, split_threads, stream (1 force row_stream, 0 never),
 * stage (1: row_stream stages rows in smem), stage_kb, portable_clusters,
 * sync (block barrier per row step), prefetch, persistent (0: one row group
 * per CTA), waves (grid = waves x resident CTAs), remat (0: buffer values read
 * after a barrier instead of recomputing, R22), tma (0: never tma_sweep, 1:
 * whenever eligible, also short sweeps), tma_rows, tma_stages, tma_teams
 * (bulk-copy ring shape), tma_team (1: row teams fed by bulk copies).  Values
 * a template cannot use are ignored.  The plan is a pure function of
 * (graph, desc, tuning): the library reads no environment variables for
 * planning or code generation.  describe() reports the string.
 * Errors: as astitch_plan, plus ERR_INVALID_ARGUMENT for an unknown key or a
 * non-integer value. */
astitch_status astitch_plan_ex(astitch_graph_t g, const astitch_plan_desc* desc, const char* tuning,
                               astitch_plan_t* out);
astitch_status astitch_plan_destroy(astitch_plan_t p);
/* Directory of the on-disk cubin cache (generated kernels compiled by NVRTC,
 * one file per source: "<dir>/<64-bit hash>.cubin", written atomically).
 * NULL or "" disables it.  Default: $XDG_CACHE_HOME/astitch, else
 * $HOME/.cache/astitch.  A cache hit skips NVRTC; describe()'s plan_time_ms
 * reports the plan's analysis / codegen / NVRTC / load times and the hits. */
astitch_status astitch_set_cache_dir(const char* dir);
/* Bytes of device workspace astitch_run needs (0 if none).  Global-stage plans
 * keep their grid barrier, column partials and buffers there; plans that take
 * row tiles from a counter (tma_sweep / tma_team, R23) keep the tile
 * counter there too (reset in-kernel after its last use, so one workspace
 * serves any number of sequential runs and CUDA-graph replays). */
astitch_status astitch_plan_workspace_bytes(astitch_plan_t p, size_t* bytes);
/* JSON description: op classes, dominants, groups, schemes, mapping, grid,
 * smem, registers, kernel count, compulsory bytes.  *len = bytes needed
 * (excluding the NUL); the string is truncated to cap-1 bytes. */
astitch_status astitch_plan_describe(astitch_plan_t p, char* json, size_t cap, size_t* len);
/* Generated CUDA source of kernel k (0-based) of the plan. */
astitch_status astitch_plan_source(astitch_plan_t p, int32_t k, char* buf, size_t cap, size_t* len);
/* Compiled sm_100a cubin of kernel k (0 bytes if FLAG_NO_COMPILE). */
astitch_status astitch_plan_cubin(astitch_plan_t p, int32_t k, void* buf, size_t cap, size_t* len);
/* Number of kernels one astitch_run launches (1 unless demoted). */
astitch_status astitch_plan_kernel_count(astitch_plan_t p, int32_t* n);
/* I/O signature: number of inputs / outputs and each one's kind and dtype. */
astitch_status astitch_plan_io_count(astitch_plan_t p, int32_t* n_inputs, int32_t* n_outputs);
astitch_status astitch_plan_io(astitch_plan_t p, int32_t is_output, int32_t index,
                               astitch_kind* kind, astitch_dtype* dtype);

/* ---------------------------------------------------------------- execution */
/* Initialise a workspace once (zeroes the grid-barrier and tile-counter
 * words).  Not needed between runs: the barrier is self-resetting and the
 * tile counters are reset by the kernel that used them. */
astitch_status astitch_workspace_init(astitch_plan_t p, void* ws, void* stream);
/* Runs the plan: one stitched kernel launch (cooperative when the plan has a
 * global stage) on `stream`.  inputs/outputs are device pointers in
 * declaration order.  rows == 0 is a no-op.  Never synchronises, allocates or
 * memsets.  Concurrent runs of one plan need distinct workspaces.
 * Errors: ERR_INVALID_ARGUMENT (null / misaligned), ERR_CUDA (launch). */
astitch_status astitch_run(astitch_plan_t p, const void* const* inputs, void* const* outputs,
                           void* ws, void* stream);
/* End-to-end run from HOST buffers: async H2D of every input from host_inputs
 * into dev_inputs, astitch_run, async D2H of every output into host_outputs,
 * all on `stream` (host buffers should be pinned for asynchrony).  Does not
 * synchronise. */
astitch_status astitch_run_host(astitch_plan_t p, const void* const* host_inputs,
                                void* const* host_outputs, const void* const* dev_inputs,
                                void* const* dev_outputs, void* ws, void* stream);
/* Same result as astitch_run_host, pipelined over `chunks` row chunks (rows are
 * the independent units): chunk i+1 is copied in while chunk i is computed and
 * chunk i-1 copied out, on three internal streams forked from and joined back
 * into `stream` (PCIe is full duplex).  A column reduction accumulates its
 * totals across chunks and its consumers run once after the last chunk.
 * Host buffers must be pinned.  Falls back to astitch_run_host for plans that
 * cannot be chunked (FULL values buffered across a grid barrier, cluster-split
 * rows, sharded plans, chunks < 2).  The first call on a global plan compiles
 * its chunk kernels.  Not safe to call concurrently on one plan. */
astitch_status astitch_run_host_pipelined(astitch_plan_t p, const void* const* host_inputs,
                                          void* const* host_outputs, const void* const* dev_inputs,
                                          void* const* dev_outputs, void* ws, void* stream,
                                          int32_t chunks);

/* ---------------------------------------------------------------- multi-GPU
 * Row-sharded execution (BASELINE north_star (4)): each process owns a
 * contiguous row range and a plan built with shard_rank / shard_world.
 * Row-local subgraphs need no communication.  Column reductions are combined
 * with one ncclAllReduce per column reduction (fp32 sum, or int32 max of
 * order keys for RMAX) of the per-rank partials on `stream`,
 * then the column consumers run in a small epilogue kernel. */
astitch_status astitch_comm_unique_id(uint8_t id[128]);
astitch_status astitch_comm_create(int32_t world, int32_t rank, const uint8_t id[128],
                                   int32_t device, astitch_comm_t* out);
astitch_status astitch_comm_destroy(astitch_comm_t c);
astitch_status astitch_run_sharded(astitch_plan_t p, astitch_comm_t c, const void* const* inputs,
                                   void* const* outputs, void* ws, void* stream);
/* The two halves of astitch_run_sharded around the collective, for callers
 * that combine the partials themselves (another collective library, or a
 * single-GPU "virtual shards" check):
 *   stage 0: stitched kernel over the shard's rows; leaves the rank-local fp32
 *            column totals at ws + offset (ncolred x cols floats, see below);
 *   stage 1: column consumers (+ the FULL sweep after the barrier) reading the
 *            combined totals from the same place.
 * astitch_plan_colpart reports the byte offset in ws and the 4-byte word
 * count: ncolred slots of `cols` words each, slot q in the order
 * astitch_plan_colpart_ops reports.  A SUM slot holds fp32 column totals
 * (combine: fp32 sum across ranks); an RMAX slot holds int32 ORDER KEYS of
 * the fp32 column maxima (combine: int32 max across ranks) -- the key is
 * monotone in the float order with NaN canonicalised to the largest key, so
 * an integer max propagates NaN as the unsharded RMAX does (reading R12),
 * which an fp32 max (ncclMax) would not.  astitch_run_sharded does exactly
 * this with ncclAllReduce(ncclFloat32, ncclSum) / (ncclInt32, ncclMax).
 * Plans without a column reduction: stage 0 = astitch_run, stage 1 = no-op. */
astitch_status astitch_run_shard_stage(astitch_plan_t p, int32_t stage, const void* const* inputs,
                                       void* const* outputs, void* ws, void* stream);
astitch_status astitch_plan_colpart(astitch_plan_t p, size_t* byte_offset, size_t* count);
/* The combine each colpart slot needs: ops[q] = ASTITCH_SUM or ASTITCH_RMAX.
 * *n = the number of column reductions (always written); ops may be NULL only
 * when that is 0; cap < *n -> ASTITCH_ERR_INVALID_ARGUMENT. */
astitch_status astitch_plan_colpart_ops(astitch_plan_t p, int32_t* ops, size_t cap, size_t* n);
/* Fused sharded run: the column-reduction exchange happens
 * INSIDE the stitched kernel over peer memory instead of an ncclAllReduce +
 * epilogue launch.  Each rank owns an exchange buffer (astitch_peer_create:
 * device memory, ~1 KB + 2 x world x ncolred x cols fp32, zeroed once) and maps
 * every other rank's buffer: astitch_peer_open with that rank's 64-byte CUDA IPC
 * handle (one process per GPU; peer access over NVLink / NVSwitch), or
 * astitch_peer_link with its peer object (several ranks in one process, e.g.
 * virtual ranks on one GPU).  astitch_run_fused then launches ONE cooperative
 * kernel per rank: sweep -> block column partials -> grid barrier -> rank-local
 * totals stored into slot [run parity][rank] of every rank's buffer (plain P2P
 * stores) -> system fence -> grid barrier -> one release flag per rank -> wait
 * for all ranks' flags of this run -> fixed-order (rank 0..world-1) combine ->
 * column consumers (+ the FULL sweep after the barrier).  Results are bitwise
 * identical on every rank.  Every rank must make the same sequence of
 * astitch_run_fused calls; the ranks' kernels must be able to run at the same
 * time (separate GPUs, or grids that fit together).  A rank that does not
 * arrive within 5 s makes the waiting kernels give up (no hang): their
 * outputs are then invalid and astitch_peer_status reports timed_out = 1.
 * Errors: ERR_INVALID_ARGUMENT (mismatched plan / peer, peer not mapped),
 * ERR_UNSUPPORTED (> 64 ranks), ERR_CUDA (allocation, IPC, launch). */
typedef struct astitch_peer_s* astitch_peer_t;
astitch_status astitch_peer_create(astitch_plan_t p, astitch_peer_t* out, uint8_t ipc_handle[64]);
astitch_status astitch_peer_open(astitch_peer_t x, int32_t rank, const uint8_t ipc_handle[64]);
astitch_status astitch_peer_link(astitch_peer_t x, int32_t rank, astitch_peer_t other);
/* Synchronous read of the buffer's error word (1 = a wait timed out). */
astitch_status astitch_peer_status(astitch_peer_t x, int32_t* timed_out);
astitch_status astitch_peer_destroy(astitch_peer_t x);
astitch_status astitch_run_fused(astitch_plan_t p, astitch_peer_t x, const void* const* inputs,
                                 void* const* outputs, void* ws, void* stream);
/* End-to-end sharded run from HOST buffers (the rank's row slice): async H2D
 * of every input into dev_inputs, then astitch_run_fused (x != NULL) or
 * astitch_run_sharded (comm c), then async D2H of every output, all on
 * `stream`.  Same errors as those calls. */
astitch_status astitch_run_sharded_host(astitch_plan_t p, astitch_comm_t c, astitch_peer_t x,
                                        const void* const* host_inputs, void* const* host_outputs,
                                        const void* const* dev_inputs, void* const* dev_outputs, void* ws,
                                        void* stream);
/* Contiguous row partition: rows_k = floor(R/g) (+1 for the first R mod g ranks). */
astitch_status astitch_shard_rows(int64_t rows, int32_t world, int32_t rank, int64_t* row_begin,
                                  int64_t* row_count);

/* ---------------------------------------------------------------- measurement aids
 * Global-barrier micro-benchmark (Table 6): launches ONE kernel of
 * `blocks` x `threads` containing `iters` grid barriers and nothing else
 * (cooperative launch).  ws needs 256 bytes, zeroed once.  Timing is the
 * caller's (CUDA events on `stream`). */
astitch_status astitch_bench_barrier(int32_t device, int32_t blocks, int32_t threads, int32_t iters,
                                     void* ws, void* stream);
/* Copy-kernel ceiling: dst[0:bytes) = src[0:bytes) with the same 128-bit
 * streaming loads/stores as the stitched kernels (bytes % 16 == 0). */
astitch_status astitch_bench_copy(int32_t device, const void* src, void* dst, size_t bytes,
                                  void* stream);

#ifdef __cplusplus
}
#endif
#endif /* ASTITCH_H_ */
