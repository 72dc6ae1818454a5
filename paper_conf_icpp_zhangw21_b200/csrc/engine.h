// engine.h -- host-side runtime: context, device arena, tensor maps, the hot-path ops,
// the in-core recursion and the out-of-core executor.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <functional>
#include <initializer_list>
#include <map>
#include <string>
#include <vector>

#include "../../include/rgsqr.h"
#include "kernels.h"

namespace rgsqr {

struct Options {
  int64_t leaf_width = 64;
  int64_t tile_rows_min = 4096;
  int64_t tile_rows_max = 16384;
  int64_t ring_depth = 3;
  int64_t algo = 0;          // 0 recursive, 1 blocked
  int64_t block_cols = 8192;
  int64_t serialize = 0;
  int64_t reuse = 1;
  int64_t leaf_ctas = 0;
  int64_t splitk = 0;
  int64_t profile = 0;
  int64_t reorth = 0;        // CGS2 (RGSQR_OPT_REORTH)
  int64_t prefetch = 1;      // OOC: upload the first ring tiles during the left child (RGSQR_OPT_PREFETCH)
  int64_t fuse_small = 1;    // fused kernel for nodes with w1, w2 <= 64 (RGSQR_OPT_FUSE_SMALL)
  int64_t split_pct = 50;    // OOC split: left child width in % (RGSQR_OPT_SPLIT_PCT; 50 = halves, the paper)
  int64_t x3_chain = 2;      // TF32X3: k-blocks per tensor-core accumulation chain (RGSQR_OPT_X3_CHAIN; 0 = unbounded)
  int64_t colchunk = 1;      // column-chunked OOC node (RGSQR_OPT_COLCHUNK, R26)
  int64_t chunk_mib = 32;    // host-path column upload chunk (RGSQR_OPT_CHUNK_MIB)
  int64_t vshards = 1;       // virtual row shards on one GPU (RGSQR_OPT_VSHARDS, device path)
  int64_t phasea_pct = 50;  // column-chunked node: % of the right child's first half projected before it
  int64_t defer_pieces = 0;  // deferred products in ~1/p of the node's A2 (RGSQR_OPT_DEFER_PIECES; 0 = upload chunks)
  int64_t graph = 1;         // replay repeated calls as CUDA graphs (RGSQR_OPT_GRAPH, graph.cu)
  int64_t eager_pct = 50;    // column-chunked node: the external projection is completed once the right
                             // child's leaves reach this % of its left half (RGSQR_OPT_EAGER_PCT)
};

struct TimedSeg {
  int kind;                  // 0 h2d, 1 d2h, 2 compute
  cudaEvent_t a, b;
};

struct GraphEntry {         // an instantiated factorization schedule (graph.cu)
  std::vector<int64_t> key;
  cudaGraphExec_t exec = nullptr;
  unsigned cnt0[2] = {0, 0}, cnt1[2] = {0, 0};   // barrier counters at capture start / end
  rgsqr_stats stats{};
  size_t arena_high = 0;     // arena high-water mark of the captured schedule
  std::vector<TimedSeg> segs;             // RGSQR_TIMELINE: the schedule's timed segments (external
  std::vector<cudaEvent_t> tl_events;     //   event record nodes) and the events they own
  uint64_t last_use = 0;
};

struct KernSeg {
  int kind;                  // 0 leaf, 1 inner, 2 outer, 3 other
  cudaEvent_t a, b;
  double flops, bytes;
};

// Bump allocator over one cudaMalloc of at most the budget; LIFO release by mark.
struct Arena {
  char* base = nullptr;
  size_t size = 0;             // this call's budget (the planner sees exactly this much)
  size_t phys = 0;             // bytes actually allocated (a reused allocation may be larger)
  size_t top = 0;
  size_t high = 0;
  void* alloc(size_t bytes) {
    size_t off = (top + 255) & ~size_t(255);
    if (off + bytes > size) return nullptr;
    top = off + bytes;
    if (top > high) high = top;
    return base + off;
  }
  size_t mark() const { return top; }
  void release(size_t m) { top = m; }
  size_t free_bytes() const { return size > top ? size - ((top + 255) & ~size_t(255)) : 0; }
};


struct Ctx {
  int device = 0;
  int rank = 0, nranks = 1;
  int num_sms = 148;
  cudaStream_t st_user = nullptr;   // set by rgsqr_set_stream
  cudaStream_t st_own = nullptr;
  cudaStream_t st_h2d = nullptr, st_d2h = nullptr, st_d2r = nullptr;   // copies: in, Q out, R out
  cudaStream_t st_h2d2 = nullptr;   // second upload queue (small uploads that must not queue behind prefetches)
  Options opt;
  rgsqr_stats stats{};
  std::string last_error;
  Arena arena;
  size_t arena_alloc_size = 0;
  // small persistent device buffers (leaf barrier/partials, breakdown flag)
  float* d_partials = nullptr;
  float* d_sn_partials = nullptr;   // fused bottom node: [LEAF_MAX_G][64 x 64] partials (128-wide: arena)
  void* d_shape = nullptr;          // distributed shape / budget agreement (3 int64)
  size_t ctx_bytes = 0;             // all context-lifetime device bytes (count against every budget)
  void* d_sn_r12op = nullptr;       // fused bottom node: 64 x 64 operand copy
  unsigned int* d_counter = nullptr;        // [0] leaf round-0 barrier, [16] fused node barriers
  unsigned int counter_host[2] = {0, 0};     // their values after every enqueued barrier (never reset)
  unsigned int leaf_epoch = 0;
  int* d_breakdown = nullptr;
  void* nccl_comm = nullptr;
  // leaf fixed-point exchange (never reset; see leaf.cu)
  unsigned long long* d_xw = nullptr;        // this GPU's words [2][LEAF_MAX_W+2]
  unsigned long long* d_xprev = nullptr;     // last-seen words, persistent
  unsigned long long** d_peers = nullptr;    // [nranks] every GPU's d_xw (IPC-mapped)
  std::vector<void*> ipc_opened;             // peer mappings to close
  float* d_r0buf = nullptr;                  // round-0 vector of a row-sharded leaf
  int64_t m_global = 0;                      // total rows of the current factorization
  std::vector<TimedSeg> segs;
  std::vector<KernSeg> ksegs;
  std::vector<cudaEvent_t> event_pool;
  size_t event_next = 0;
  bool timing = false;
  // a leaf exchange timed out (a rank did not arrive): late contributions may still land in the
  // never-reset exchange words, so the handle refuses further factorizations (rgsqr_destroy it)
  bool broken = false;
  std::vector<GraphEntry> graphs;            // captured schedules (RGSQR_OPT_GRAPH)
  uint64_t graph_clock = 0;
  int64_t n_graph_captures = 0;
  bool graph_failed = false;                 // capture not supported here: eager launches from then on
  bool capturing = false;                    // inside a stream capture (no timing events)
  std::vector<cudaEvent_t> capture_events;   // fresh events handed out during a capture
  bool graph_timeline = false;               // capture timing segments (RGSQR_TIMELINE)
  std::vector<cudaEvent_t> graph_tl_events;  // their events (moved into the graph entry)
  std::vector<std::vector<int64_t>> graph_bad;   // signatures whose capture failed: eager
  std::map<void*, size_t> host_allocs;       // rgsqr_host_alloc buffers (NUMA-placed, registered)
  int host_numa_node = -1;                   // the GPU's NUMA node (-1: unknown / single node)

  cudaStream_t compute() const { return st_user ? st_user : st_own; }
  cudaEvent_t ev();
  // per-launch profiling (RGSQR_OPT_PROFILE)
  cudaEvent_t kbegin(cudaStream_t st) {
    if (!opt.profile) return nullptr;
    cudaEvent_t e = ev();
    cudaEventRecord(e, st);
    return e;
  }
  void kend(int kind, cudaStream_t st, cudaEvent_t a, double flops, double bytes) {
    if (!a) return;
    cudaEvent_t b = ev();
    cudaEventRecord(b, st);
    ksegs.push_back({kind, a, b, flops, bytes});
  }
  void begin_call() {           // reset per-call accounting
    segs.clear();
    ksegs.clear();
    event_next = 0;
  }
  void collect_kernel_stats();  // after a synchronize
};

// CUDA-graph replay (graph.cu)
std::vector<int64_t> graph_key(Ctx* c, int kind, std::initializer_list<int64_t> call);
bool graph_allowed(Ctx* c);
GraphEntry* graph_find(Ctx* c, const std::vector<int64_t>& key);
bool graph_known_bad(Ctx* c, const std::vector<int64_t>& key);
void graph_drop_all(Ctx* c);
int graph_capture_begin(Ctx* c, cudaStream_t st, unsigned cnt0[2]);
int graph_capture_end(Ctx* c, cudaStream_t st, std::vector<int64_t> key, const unsigned cnt0[2], int rc,
                      GraphEntry** out);
int graph_launch(Ctx* c, GraphEntry* g, cudaStream_t st);

// status helpers
int fail(Ctx* c, int status, const std::string& msg);
#define RGSQR_CUDA(c, call)                                                        \
  do {                                                                             \
    cudaError_t _e = (call);                                                       \
    if (_e != cudaSuccess)                                                         \
      return fail((c), RGSQR_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(_e)); \
  } while (0)

int elem_bytes(int precision);
bool encode_tmap_2d(CUtensorMap* map, int precision, const void* base, uint64_t inner, uint64_t outer,
                    uint64_t outer_stride_bytes, uint32_t box_inner, uint32_t box_outer, std::string* err,
                    int swz = 0);  // 0 SWIZZLE_128B, 1 SWIZZLE_128B_ATOM_32B, 2 none

// ---- ops (device pointers, on stream st) ----
// reduce_ranks: in a row-sharded run, sum the R12 partials of all ranks (NCCL) before the
// operand copy is formed; the streamed inner product passes false per tile and reduces
// once after its last tile (reduce_r12).
int op_inner(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m,
             int64_t w1, int64_t w2, float* R12, int64_t ldr, void* R12op, int64_t ldop, int accumulate,
             cudaStream_t st, bool reduce_ranks = true);
int reduce_r12(Ctx* c, int prec, float* R12, int64_t ldr, void* R12op, int64_t ldop, int64_t w1, int64_t w2,
               cudaStream_t st);
int sync_shape(Ctx* c, int64_t m, size_t* budget);
// NCCL (loaded at run time); sum-allreduce in place on stream st
int nccl_allreduce(Ctx* c, void* buf, size_t count, int nccl_dtype, cudaStream_t st);
constexpr int NCCL_INT64 = 4, NCCL_FLOAT32 = 7, NCCL_FLOAT64 = 8;
int op_outer(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* R12op, int64_t ldr, void* A2,
             int64_t lda, int64_t m, int64_t w1, int64_t w2, cudaStream_t st);
int op_leaf(Ctx* c, int prec, void* P, int64_t ldp, int64_t m, int64_t w, float* R11, int64_t ldr,
            int64_t col_offset, cudaStream_t st, bool r0_pre = false);
int leaf_width_for(Ctx* c, int64_t m);
int64_t split_width(int64_t w, int64_t leaf);

// ---- factorizations ----
size_t incore_workspace_bytes(Ctx* c, int prec, int64_t m, int64_t n);
// Optional callbacks of the in-core recursion, used by the out-of-core executor to
// overlap a node's column upload / Q download with its factorization:
//   need(c)      -- called before any op that reads columns [0, c) of the node
//   leaf_done(c) -- called after the leaf ending at column c (Q[:, 0:c) is final)
// A deferred projection against a Q1 that is NOT part of the node (the left child of an
// out-of-core parent, resident in HBM): for node columns [0, end), R12 = Q1^T A2 and
// A2 -= Q1 R12 (Eq. 2), applied chunk by chunk before the node's own deferred
// products (ancestor first), R12 handed to r_out (downloaded to the host R) per chunk.
struct ExtProduct {
  const void* Q1 = nullptr;
  int64_t ldq = 0, w1 = 0;
  int64_t end = 0;                            // node columns [0, end) receive the product
  int64_t applied = 0;
  int64_t piece = 0;                          // columns per application (0: the upload chunk)
  float* R12[2] = {nullptr, nullptr};         // w1 x piece fp32, alternating (R12[1] may be null)
  cudaEvent_t free_ev[2] = {nullptr, nullptr};  // R12[i] may be overwritten after this event
  void* R12op = nullptr;                      // w1 x piece, operand type
  int n_done = 0;
  std::function<cudaEvent_t(int64_t a, int64_t b, const float* R12)> r_out;  // download; event after it
  std::function<void()> done;                 // after the last chunk: Q1 is dead once sc gets there
};

struct IncoreHooks {
  std::function<void(int64_t)> need;          // make the compute stream wait for columns < col_end
  std::function<void(int64_t)> leaf_done;     // columns < col_end are final
  std::function<bool(int64_t)> pending;       // need(col_end) would still wait on an upload
  int64_t chunk = 0;                          // upload chunk width (columns)
  ExtProduct* ext = nullptr;                  // optional projection against an external Q1
};
int apply_ext(Ctx* c, int prec, char* A, int64_t lda, int64_t m, IncoreHooks* hk, int64_t upto, cudaStream_t st);
int incore_factor(Ctx* c, int prec, void* A, int64_t lda, int64_t m, int64_t n, float* R, int64_t ldr,
                  int64_t col_offset, cudaStream_t st, IncoreHooks* hooks = nullptr);
int factor_device(Ctx* c, const void* A, int64_t lda, int64_t m, int64_t n, void* Q, float* R, int prec,
                  size_t budget);
int factor_host(Ctx* c, const void* A, int64_t lda, int64_t m, int64_t n, void* Q, float* R, int prec,
                size_t budget);
int ooc_gemm(Ctx* c, int op, int tiling, int64_t block, const void* Q1, int64_t ldq, void* A2, int64_t lda,
             float* R12, int64_t ldr, int64_t m, int64_t w1, int64_t w2, int prec, size_t budget);

}  // namespace rgsqr
