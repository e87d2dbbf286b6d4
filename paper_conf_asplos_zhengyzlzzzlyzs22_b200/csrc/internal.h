// Internal data structures of the AStitch B200 engine (not part of the C ABI).
//
//   Graph    — the tiny SSA op-graph IR of one stitch op (Sec. 4.1).
//   Analysis — per-op class, dominant / group, scheme (Sec. 4.3).
//   Mapping  — the adaptive thread mapping chosen for the dominant schedule
//              (task packing / splitting).
//   Plan     — everything astitch_run needs: kernels, launch config, workspace.
#pragma once

#include <algorithm>
#include <cstdint>
#include <memory>
#include <string>
#include <vector>

#include "astitch.h"

namespace astitch {

// ------------------------------------------------------------------ errors
void set_error(const std::string& msg);
astitch_status fail(astitch_status s, const std::string& msg);

struct Error {
  astitch_status status;
  std::string msg;
};

// ------------------------------------------------------------------ IR
enum class NodeType { Input, Const, Unary, Binary, Reduce, Bcast };

struct Node {
  NodeType type = NodeType::Input;
  int sub = 0;             // unop / binop / redop
  int axis = 0;            // astitch_axis for Reduce / Bcast
  int a = -1, b = -1;      // operands
  astitch_kind kind = ASTITCH_FULL;
  astitch_dtype dtype = ASTITCH_F32;  // storage dtype (inputs)
  double cval = 0.0;       // Const value
  int input_index = -1;    // position in the input list
};

struct Graph {
  std::vector<Node> nodes;
  std::vector<int> inputs;                  // node ids in input order
  std::vector<int> outputs;                 // node ids in output order
  std::vector<astitch_dtype> output_dtypes;
  int lengths_node = -1;
  int64_t rows_per_segment = 0;
  int segments_node = -1;                   // packed varlen table (astitch_graph_segments)
  int nseg = 0;
  int64_t seg_elems = 0;                    // elements of every FULL tensor when ragged
};

int dtype_size(astitch_dtype d);
const char* dtype_name(astitch_dtype d);
const char* kind_name(astitch_kind k);
const char* unop_name(int op);
const char* binop_name(int op);

// ------------------------------------------------------------------ analysis
// Op classes of the paper's taxonomy: light / heavy element-wise,
// broadcast, row- / column-reduce.
enum class OpClass { Input, Const, LightEW, HeavyEW, BcastRow, BcastCol, ReduceRow, ReduceCol };
// Stitching schemes of Table 1.
enum class Scheme { Independent, Local, Regional, Global };

const char* opclass_name(OpClass c);
const char* scheme_name(Scheme s);

struct NodeInfo {
  OpClass cls = OpClass::Input;
  bool live = false;           // reaches an output
  bool post = false;           // depends on a column reduction (after the grid barrier)
  int level = 0;               // number of column reductions (grid barriers) on its path
  bool candidate = false;      // dominant candidate (Step 1)
  bool dominant = false;       // final dominant
  bool sub_dominant = false;
  int group = -1;              // op group id
  Scheme scheme = Scheme::Local;
  bool global_full = false;    // FULL value buffered in HBM across the barrier
  bool precise_col = false;    // cancellation-prone column value: fp64 sum, applied as hi+lo (R7c)
  unsigned remat_mask = 0;     // bit L: FULL value recomputed in the sweep of level L (instead of an HBM buffer)
  std::vector<int> consumers;
};

enum class Template {
  RowTeam,     // row-reduce / EW: a team of lanes per row, registers + shuffles (regional)
  PackedTile,  // many tiny rows: TMA-bulk tiles in smem, thread per row (horizontal packing)
  GlobalSweep, // column reduce: vertical packing + block partials + grid barrier (global)
  SplitRow,    // few long rows: row split over a thread-block cluster (task splitting)
  RowStream    // rows longer than a team's registers: column tiles, one pass per row-reduction level
};
const char* template_name(Template t);

struct Mapping {
  Template tmpl = Template::RowTeam;
  int vec_elems = 1;        // E: elements per chunk (one vector access per tensor)
  int chunks = 1;           // C / E
  int team = 32;            // T: lanes cooperating on one row
  int chunks_per_lane = 1;  // V
  int threads = 256;        // block size
  int rows_per_block = 8;   // teams per block (threads / T), or tile rows (PackedTile)
  int row_unroll = 1;       // U: rows per team per iteration (vertical packing ILP)
  bool prefetch = true;     // software-pipeline the next row's loads
  int single_wave_bps = 0;  // RowTeam: blocks/SM that give every row its own team in one wave (0 = off)
  bool sync_steps = false;  // block barrier at every row step of a persistent sweep (keeps the CTA's warps aligned)
  bool nonpersistent = false;  // RowTeam: one row group per CTA (the block scheduler orders the sweep)
  int grid_waves = 0;       // PackedTile / RowTeam: grid = waves x resident CTAs (0 = the planner decides)
  int nslab = 1;            // GlobalSweep: column slabs of T x V x E columns (wide rows); CTA b owns slab b % nslab
  bool hoist_colvec = true; // keep COLVEC operands in registers across rows
  int tile_rows = 0;        // PackedTile rows per stage
  int stages = 0;           // PackedTile pipeline stages
  int split = 1;            // CTAs per row (task splitting; 1 = none)
  bool stage_row = false;   // row_stream: the row's inputs staged in shared memory (regional)
  int64_t grid = 1;
  int blocks_per_sm = 1;    // assume-relax-apply target
  int reg_cap = 255;
  int64_t vertical_trips = 1;
  double lane_util = 1.0;
  int smem_bytes = 0;       // dynamic shared memory per block
  // GlobalSweep as tma_sweep: row tiles of tma_rows rows staged in a ring of
  // tma_stages shared-memory stages by bulk copies (UBLKCP) that one producer
  // warp issues for tiles taken from a workspace counter (address order);
  // rows_per_block teams of T lanes compute from shared memory; column sums
  // in exact binned accumulators (order-independent, reading R23)
  bool tma_sweep = false;
  // RowTeam as tma_team: the same producer warp / bulk-copy ring / address-
  // ordered tiles for row-wise plans; one bulk copy per row (its valid prefix)
  bool tma_team = false;
  int tma_rows = 0;
  int tma_stages = 0;
  int bank_conflict_ways = 1;
  std::string reason;       // selector decision trace
};

// ------------------------------------------------------------------ tuning
// Explicit overrides of the planner's choices (astitch_plan_ex's tuning
// string "key=value,..."; experiments and tests).  0 / -1 = the planner
// decides.  A plan is a pure function of (graph, desc, tuning): the library
// reads no environment variables for planning or code generation.
struct Tuning {
  int threads = 0;          // block size
  int unroll = 0;           // rows per team per iteration (U)
  int team = 0;             // lanes per row (row-wise plans)
  int bps = 0;              // fixed blocks-per-SM target (no assume-relax-apply bisection)
  int vec_bytes = 0;        // 16 or 32: vector width of a chunk
  int hoist = -1;           // 1 / 0: keep COLVEC operands in registers (or re-read per row)
  int tile_stages = 0, tile_rows = 0, tile_threads = 0;  // packed_tile pipeline
  int split = 0, split_threads = 0;                       // split_row cluster size / CTA size
  int stream = -1;          // 1: force row_stream, 0: never stream
  int stage = 0;            // 1: row_stream stages the row's inputs in smem
  int stage_kb = 0;         // row_stream staging budget per CTA (KB)
  int portable_clusters = 0;  // 1: never ask for 16-CTA clusters
  int sync = -1;            // 1 / 0: block barrier at every row step of a persistent sweep
  int prefetch = -1;        // 1: software-prefetch the next rows in the global sweep (off by default)
  int persistent = -1;      // 0: row teams on a non-persistent grid (one row group per CTA)
  int waves = 0;            // packed tiles: grid = waves x the resident CTAs
  int remat = -1;           // 0: buffer every FULL value read after a barrier in HBM (no recomputation)
  int tma = -1;             // 0: never plan a global sweep as tma_sweep, 1: whenever eligible (default)
  int tma_team = -1;        // 1: row-team plans as tma_team, 0: never
  int tma_rows = 0, tma_stages = 0, tma_teams = 0;  // tma_sweep tile rows / ring stages / compute teams
  std::string text;         // the string it was parsed from (describe())
};
bool parse_tuning(const char* s, Tuning& t, std::string& err);

// ------------------------------------------------------------------ plan
struct Kernel {
  std::string name;
  std::string source;
  std::vector<char> cubin;
  std::string log;
  int threads = 256;
  int64_t grid = 1;
  int smem = 0;
  bool cooperative = false;
  bool pdl = false;          // programmatic dependent launch attribute
  int regs = -1;
  int spill_bytes = -1;
  int occupancy = -1;        // blocks per SM from the occupancy API
  int cluster = 1;           // CTAs per cluster (compile-time __cluster_dims__)
  int max_clusters = -1;     // co-resident clusters (cuOccupancyMaxActiveClusters), cluster kernels
  void* module = nullptr;    // CUmodule
  void* function = nullptr;  // CUfunction
};

struct WsLayout {
  size_t barrier = 0;        // 2 x u32 (+ pad)
  size_t partials = 0;       // [grid][ncolred][C] fp32 block partials
  size_t colvals = 0;        // [ncolvec_post][C] fp32 finalized column values
  size_t globals = 0;        // [nglobal_full][R][C] fp32 buffers
  size_t total = 0;
};

struct Plan {
  Graph g;
  astitch_plan_desc desc{};
  Tuning tune;
  int sm_count = 148;
  int smem_optin = 232448;       // max dynamic+static smem per block (B200: 227 KB; device query)
  std::vector<std::string> demotions;  // resource-driven mapping changes (a6), in order (describe())
  // plan (JIT) time, milliseconds: analysis + mapping, code generation,
  // NVRTC (or cubin cache), module load; and the compile / cache counts
  double ms_analyse = 0, ms_codegen = 0, ms_nvrtc = 0, ms_load = 0, ms_total = 0;
  int n_compiles = 0, n_mem_hits = 0, n_disk_hits = 0;
  std::vector<NodeInfo> info;
  std::vector<std::vector<int>> groups;
  Mapping map;
  std::vector<int> colreds;      // column reduce node ids (in order)
  std::vector<int> post_colvecs; // COLVEC values computed after the barrier (incl. colreds)
  int n_precise_colreds = 0;     // column sums with an extra lo partial slot (reading R7c)
  std::vector<int> global_fulls; // FULL / ROWVEC values buffered in HBM across a barrier
  std::vector<size_t> gbuf_off;  // byte offset of each one's buffer within ws.globals (a6 reuse)
  int gbuf_slots = 0;            // distinct buffers after liveness-based reuse
  bool needs_sweep2 = false;     // FULL / ROWVEC work after the (first) grid barrier
  int max_level = 0;             // grid barriers needed by dependent column reductions
  bool stream_fallback = false;  // registers overflowed at 1 block/SM: stream the rows
  bool portable_clusters = false; // 16-CTA clusters not co-resident in one wave: plan with <= 8
  std::vector<Kernel> kernels;   // kernels launched by astitch_run, in order
  std::vector<Kernel> shard_kernels; // kernels of the sharded path (after the allreduce)
  std::vector<Kernel> fused_kernels; // fused sharded path (P2P exchange in-kernel), built lazily
  // chunked host pipeline (astitch_run_host_pipelined): copy-in / compute /
  // copy-out streams, per-chunk events, and for global plans the row-chunk
  // kernels (shard-main with accumulation + column epilogue), built lazily
  std::vector<Kernel> chunk_kernels;
  void* pipe_streams[3] = {nullptr, nullptr, nullptr};
  std::vector<void*> pipe_events;
  WsLayout ws;
  uint64_t compulsory_bytes = 0;
  int device = -1;
  std::string describe;
};

// a cooperative kernel's grid clamped to what is co-resident (whole row groups
// of column slabs); 0 if not even one row group fits
inline int64_t resident_grid(const Plan& p, const Kernel& k) {
  int64_t g = std::min<int64_t>(k.grid, static_cast<int64_t>(k.occupancy) * p.sm_count);
  if (p.map.nslab > 1) g = (g / p.map.nslab) * p.map.nslab;
  return g;
}

// planner.cpp
void analyse(Plan& p);                 // a1, a2, a5: classes, dominants, groups, schemes
void select_mapping(Plan& p);          // a3, a4, a6, a7: thread mapping, memory, launch
void plan_workspace(Plan& p);
void retune_grid(Plan& p);
std::string describe_json(const Plan& p);
uint64_t compulsory_bytes(const Plan& p);

// codegen.cpp
std::string generate_kernel(const Plan& p, int role, const std::string& name);
enum KernelRole { ROLE_MAIN = 0, ROLE_SHARD_MAIN = 1, ROLE_SHARD_FINAL = 2, ROLE_SHARD_SWEEP2 = 3, ROLE_FUSED = 4 };

// Peer exchange buffer of the fused sharded run (astitch_run_fused), one per
// rank, device memory:  [peers: world x u64 device addresses of every rank's
// buffer as mapped in this process] [flags: world x u32] [err: u32] ... then at
// kXSlots: 2 (generation parity) x world x ncolred x cols fp32 slots.
constexpr size_t kXFlags = 8 * 64;           // up to 64 ranks
constexpr size_t kXErr = kXFlags + 4 * 64;
constexpr size_t kXGen = kXErr + 4;          // u32: generation of the last fused run (bumped in-kernel)
constexpr size_t kXSlots = 1024;
inline size_t xbuf_bytes(int world, size_t ncolred, int64_t cols) {
  return kXSlots + 2 * static_cast<size_t>(world) * ncolred * static_cast<size_t>(cols) * 4;
}

// jit.cpp
// cache_state (optional out): 0 = compiled by NVRTC, 1 = in-process cache hit,
// 2 = on-disk cache hit (astitch_set_cache_dir)
bool nvrtc_compile(const std::string& src, const std::string& name, std::vector<char>& cubin,
                   std::string& log, std::string& err, int* cache_state = nullptr);
const char* device_header_source();
void set_cache_dir(const char* dir);  // "" disables the on-disk cubin cache
bool log_enabled();                   // ASTITCH_LOG=1: plan summaries on stderr (diagnostics only)

// driver.cpp — libcuda via dlopen
struct Driver;
Driver* driver(std::string& err);
bool drv_load(Plan& p, Kernel& k, std::string& err);
bool drv_launch(const Kernel& k, void* params, size_t params_size, void* stream, std::string& err);
bool drv_launch_args(const Kernel& k, void** args, void* stream, std::string& err);
bool drv_unload(Kernel& k);
bool drv_memset_async(void* ptr, size_t bytes, void* stream, std::string& err);
bool drv_memcpy_async(void* dst, const void* src, size_t bytes, int kind, void* stream,
                      std::string& err);
bool drv_device_info(int device, int& sm_count, int& max_smem_optin, std::string& err);
bool drv_sync(void* stream, std::string& err);
bool drv_stream_create(void** s, std::string& err);
bool drv_event_create(void** e, std::string& err);
bool drv_event_record(void* e, void* s, std::string& err);
bool drv_stream_wait(void* s, void* e, std::string& err);
void drv_stream_destroy(void* s);
bool drv_alloc_zero(int device, size_t bytes, void** ptr, std::string& err);
void drv_free(void* ptr);
bool drv_htod(void* dst, const void* src, size_t bytes, std::string& err);
bool drv_dtoh(void* dst, const void* src, size_t bytes, std::string& err);
bool drv_ipc_get(void* ptr, unsigned char handle[64], std::string& err);
bool drv_ipc_open(int device, const unsigned char handle[64], void** ptr, std::string& err);
void drv_ipc_close(void* ptr);
void drv_event_destroy(void* e);

// kernel parameter block (mirrors the struct emitted by codegen)
constexpr int kMaxIO = 16;
struct KernelParams {
  const void* in[kMaxIO];
  void* out[kMaxIO];
  void* ws;
  long long rows;
  long long row_offset;   // global row index of row 0 (chunked runs; mask segments)
  int flags;              // bit 0: accumulate column totals onto earlier chunks
  void* xbuf;             // fused sharded run: this rank's peer exchange buffer
  unsigned int gen;       // unused (the fused run's generation lives in the exchange buffer)
};

}  // namespace astitch

struct astitch_graph_s {
  astitch::Graph g;
};
struct astitch_plan_s {
  std::unique_ptr<astitch::Plan> p;
};
