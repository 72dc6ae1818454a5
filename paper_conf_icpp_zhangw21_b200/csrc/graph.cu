// graph.cu -- CUDA-graph replay of whole factorizations (RGSQR_OPT_GRAPH).
//
// A factorization's schedule is a pure function of (buffers, shape, precision, budget, options):
// the executor's host logic only decides which copies and kernels to enqueue on which stream.
// The first call with a given signature is stream-captured (every stream the executor uses is
// forked from and joined back into the compute stream), later calls replay the instantiated
// graph with one cudaGraphLaunch.  Measured reason (R30): with the host link busy,
// every eagerly launched kernel waits longer for its command to reach the GPU -- the kernels
// of the out-of-core factorization took ~35% longer while copies ran beside them
// (scripts/interference.py) -- a replayed graph's work descriptors are already on the device.
//
// Replay-invariant state: the leaf's exchange words are never reset and readers difference
// against the last value seen (persisted in device memory), so replays stay consistent.  The two
// grid-barrier counters are the exception: launches bake their target values, so the graph
// first resets both counters to their values at capture time (set_counters_kernel) and the
// host copy is advanced to the end-of-graph values on every launch.
#include <algorithm>
#include <cstring>

#include "engine.h"

namespace rgsqr {

namespace {
__global__ void set_counters_kernel(unsigned* c0, unsigned v0, unsigned* c1, unsigned v1) {
  *c0 = v0;
  *c1 = v1;
}
constexpr size_t kMaxGraphs = 8;
}  // namespace

std::vector<int64_t> graph_key(Ctx* c, int kind, std::initializer_list<int64_t> call) {
  std::vector<int64_t> k;
  k.push_back(kind);
  k.insert(k.end(), call.begin(), call.end());
  k.push_back(reinterpret_cast<int64_t>(c->arena.base));
  k.push_back((int64_t)c->arena.size);
  k.push_back(reinterpret_cast<int64_t>(c->compute()));
  static_assert(sizeof(Options) % sizeof(int64_t) == 0, "Options holds int64_t fields only");
  const int64_t* o = reinterpret_cast<const int64_t*>(&c->opt);
  k.insert(k.end(), o, o + sizeof(Options) / sizeof(int64_t));
  return k;
}

bool graph_allowed(Ctx* c) {
  static const bool env_off = getenv("RGSQR_LEAF_DEBUG") || getenv("RGSQR_LEAF_DEBUG2");
  return c->opt.graph != 0 && !c->opt.profile && !c->graph_failed && c->nccl_comm == nullptr && !env_off;
}

static void destroy_entry(GraphEntry& g) {
  if (g.exec) cudaGraphExecDestroy(g.exec);
  for (cudaEvent_t e : g.tl_events) cudaEventDestroy(e);
  g.exec = nullptr;
  g.tl_events.clear();
}

bool graph_known_bad(Ctx* c, const std::vector<int64_t>& key) {
  for (auto& k : c->graph_bad)
    if (k == key) return true;
  return false;
}

GraphEntry* graph_find(Ctx* c, const std::vector<int64_t>& key) {
  for (auto& g : c->graphs)
    if (g.key == key) {
      g.last_use = ++c->graph_clock;
      return &g;
    }
  return nullptr;
}

void graph_drop_all(Ctx* c) {
  for (auto& g : c->graphs) destroy_entry(g);
  c->graphs.clear();
}

int graph_capture_begin(Ctx* c, cudaStream_t st, unsigned cnt0[2]) {
  cnt0[0] = c->counter_host[0];
  cnt0[1] = c->counter_host[1];
  cudaError_t e = cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed);
  if (e != cudaSuccess) {
    cudaGetLastError();
    c->graph_failed = true;
    return 0;   // not capturing: the caller runs eagerly
  }
  c->capturing = true;
  static const bool timeline = getenv("RGSQR_TIMELINE") != nullptr;
  c->graph_timeline = timeline;
  set_counters_kernel<<<1, 1, 0, st>>>(c->d_counter, cnt0[0], c->d_counter + 16, cnt0[1]);
  return 1;
}

int graph_capture_end(Ctx* c, cudaStream_t st, std::vector<int64_t> key, const unsigned cnt0[2], int rc,
                      GraphEntry** out) {
  *out = nullptr;
  c->capturing = false;
  cudaGraph_t g = nullptr;
  cudaError_t e = cudaStreamEndCapture(st, &g);
  cudaGraphExec_t exec = nullptr;
  if (rc >= 0 && e == cudaSuccess && g) e = cudaGraphInstantiate(&exec, g, 0);
  if (g) cudaGraphDestroy(g);
  for (cudaEvent_t ev : c->capture_events) cudaEventDestroy(ev);   // (internal edges of the graph now)
  c->capture_events.clear();
  std::vector<cudaEvent_t> tl_events;
  tl_events.swap(c->graph_tl_events);
  if (rc < 0 || e != cudaSuccess || !exec) {
    for (cudaEvent_t ev : tl_events) cudaEventDestroy(ev);
    c->segs.clear();
    // nothing captured ran: the barrier counters are where they were; the caller re-runs the
    // schedule eagerly (a genuine error, e.g. a budget too small, then surfaces from that run)
    c->counter_host[0] = cnt0[0];
    c->counter_host[1] = cnt0[1];
    if (exec) cudaGraphExecDestroy(exec);
    cudaGetLastError();
    c->graph_bad.push_back(std::move(key));
    return 0;
  }
  if (c->graphs.size() >= kMaxGraphs) {
    size_t lru = 0;
    for (size_t i = 1; i < c->graphs.size(); ++i)
      if (c->graphs[i].last_use < c->graphs[lru].last_use) lru = i;
    destroy_entry(c->graphs[lru]);
    c->graphs.erase(c->graphs.begin() + lru);
  }
  GraphEntry ge;
  ge.key = std::move(key);
  ge.exec = exec;
  ge.cnt0[0] = cnt0[0];
  ge.cnt0[1] = cnt0[1];
  ge.cnt1[0] = c->counter_host[0];
  ge.cnt1[1] = c->counter_host[1];
  ge.stats = c->stats;
  ge.arena_high = c->arena.high;
  ge.segs = c->segs;
  ge.tl_events = std::move(tl_events);
  ge.last_use = ++c->graph_clock;
  c->graphs.push_back(std::move(ge));
  *out = &c->graphs.back();
  c->n_graph_captures++;
  return 1;
}

int graph_launch(Ctx* c, GraphEntry* g, cudaStream_t st) {
  c->stats = g->stats;   // what the captured schedule enqueued (bytes, launches, nodes)
  c->stats.graph_captures = c->n_graph_captures;
  c->stats.graph_replay = 1;
  c->counter_host[0] = g->cnt1[0];
  c->counter_host[1] = g->cnt1[1];
  c->arena.high = std::max(c->arena.high, g->arena_high);
  c->segs = g->segs;   // (RGSQR_TIMELINE: the graph's own event record nodes)
  RGSQR_CUDA(c, cudaGraphLaunch(g->exec, st));
  return RGSQR_OK;
}

}  // namespace rgsqr
