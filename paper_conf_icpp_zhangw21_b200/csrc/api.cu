// api.cu -- the extern "C" boundary declared in include/rgsqr.h.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <pthread.h>
#include <sched.h>
#include <sys/mman.h>

#include <cctype>
#include <cstdio>
#include <thread>

#include <chrono>
#include <climits>
#include <cstring>
#include <new>

#include "engine.h"

using namespace rgsqr;

namespace rgsqr {

int ensure_arena(Ctx* c, size_t want) {
  if (c->arena.base && c->arena.phys >= want && c->arena.phys <= want + ((size_t)64 << 20)) {
    // reuse the allocation, but the budget stays exact: plans never depend on call history
    c->arena.size = want;
    c->arena.top = 0;
    c->arena.high = 0;
    return RGSQR_OK;
  }
  if (c->arena.base) {
    graph_drop_all(c);   // (captured schedules address the old arena)
    cudaFree(c->arena.base);
    c->arena = Arena{};
  }
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, want);
  if (e != cudaSuccess)
    return fail(c, RGSQR_ERR_CUDA, "arena cudaMalloc(" + std::to_string(want) + "): " + cudaGetErrorString(e));
  c->arena.base = static_cast<char*>(p);
  c->arena.size = want;
  c->arena.phys = want;
  c->arena.top = 0;
  c->arena.high = 0;
  return RGSQR_OK;
}

size_t resolve_budget(Ctx* c, size_t budget) {
  if (budget != 0) return budget;
  size_t fr = 0, tot = 0;
  cudaMemGetInfo(&fr, &tot);
  size_t mine = c->arena.base ? c->arena.phys : 0;
  size_t avail = fr + mine;
  const size_t reserve = (size_t)512 << 20;
  return avail > reserve ? avail - reserve : avail / 2;
}

void reset_stats(Ctx* c) {
  std::memset(&c->stats, 0, sizeof(c->stats));
  c->stats.first_breakdown_col = -1;
}

int validate(Ctx* c, const void* A, int64_t lda, int64_t m, int64_t n, const void* Q, int prec) {
  if (!A || !Q) return fail(c, RGSQR_ERR_INVALID_ARG, "null A or Q");
  if (n < 1 || m < n) return fail(c, RGSQR_ERR_INVALID_ARG, "need 1 <= n <= m");
  if (lda < m) return fail(c, RGSQR_ERR_INVALID_ARG, "need lda >= m");
  if (prec < RGSQR_FP16 || prec > RGSQR_TF32X3) return fail(c, RGSQR_ERR_INVALID_ARG, "bad precision");
  const int s = elem_bytes(prec);
  if ((lda * s) % 16 != 0) return fail(c, RGSQR_ERR_INVALID_ARG, "lda*sizeof(elem) must be a multiple of 16");
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(Q)) & 15)
    return fail(c, RGSQR_ERR_INVALID_ARG, "A and Q must be 16-byte aligned");
  return RGSQR_OK;
}

// A, Q, R in HBM; in-core recursion on Q (after copying A into Q when they differ).
int factor_device(Ctx* c, const void* A, int64_t lda, int64_t m, int64_t n, void* Q, float* R, int prec,
                  size_t budget) {
  int rc = validate(c, A, lda, m, n, Q, prec);
  if (rc < 0) return rc;
  if (!R) return fail(c, RGSQR_ERR_INVALID_ARG, "null R");
  reset_stats(c);
  c->begin_call();
  rc = sync_shape(c, m, &budget);
  if (rc < 0) return rc;
  if (c->opt.vshards > 1) {
    const int64_t p = c->opt.vshards;
    if (c->nccl_comm) return fail(c, RGSQR_ERR_UNSUPPORTED, "virtual shards need a single-GPU context");
    if (m % p != 0 || ((m / p) * elem_bytes(prec)) % 16 != 0)
      return fail(c, RGSQR_ERR_UNSUPPORTED, "virtual shards: m must split into equal 16-byte aligned row blocks");
  }
  auto t0 = std::chrono::steady_clock::now();
  const size_t ws = incore_workspace_bytes(c, prec, m, n);
  size_t cap = resolve_budget(c, budget);
  cap = cap > c->ctx_bytes ? cap - c->ctx_bytes : 0;   // context buffers count against the budget
  if (ws > cap) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "workspace " + std::to_string(ws) + " > budget");
  rc = ensure_arena(c, ws);
  if (rc < 0) return rc;
  cudaStream_t st = c->compute();
  const int s = elem_bytes(prec);
  auto schedule = [&]() -> int {
    if (Q != A)
      RGSQR_CUDA(c, cudaMemcpy2DAsync(Q, lda * s, A, lda * s, m * s, n, cudaMemcpyDeviceToDevice, st));
    RGSQR_CUDA(c, cudaMemsetAsync(R, 0, (size_t)n * n * sizeof(float), st));
    RGSQR_CUDA(c, cudaMemsetAsync(c->d_breakdown, 0x7f, sizeof(int), st));
    return incore_factor(c, prec, Q, lda, m, n, R, n, 0, st);
  };
  if (graph_allowed(c)) {
    // replay the captured schedule (graph.cu); the first call with this signature captures it
    auto key = graph_key(c, 1, {reinterpret_cast<int64_t>(A), reinterpret_cast<int64_t>(Q),
                                reinterpret_cast<int64_t>(R), lda, m, n, prec});
    GraphEntry* g = graph_find(c, key);
    if (!g && !graph_known_bad(c, key)) {
      unsigned cnt0[2];
      const size_t amark = c->arena.mark();
      if (graph_capture_begin(c, st, cnt0)) {
        const int src = schedule();
        graph_capture_end(c, st, std::move(key), cnt0, src, &g);
        if (!g) {   // capture failed: nothing ran, re-run eagerly
          c->arena.release(amark);
          reset_stats(c);
        }
      }
    }
    rc = g ? graph_launch(c, g, st) : schedule();
  } else {
    rc = schedule();
  }
  if (rc < 0) return rc;
  int brk = INT_MAX;
  RGSQR_CUDA(c, cudaMemcpyAsync(&brk, c->d_breakdown, sizeof(int), cudaMemcpyDeviceToHost, st));
  RGSQR_CUDA(c, cudaStreamSynchronize(st));
  auto t1 = std::chrono::steady_clock::now();
  c->stats.wall_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
  c->stats.arena_bytes = (int64_t)c->arena.size;
  c->stats.arena_high_water = (int64_t)c->arena.high;
  c->stats.ctx_device_bytes = (int64_t)c->ctx_bytes;
  c->stats.flops = (int64_t)(2.0 * m * (double)n * n);
  if (brk == -2) {
    c->broken = true;
    return fail(c, RGSQR_ERR_CUDA, "leaf exchange timed out (a rank did not arrive)");
  }
  c->stats.first_breakdown_col = brk == 0x7f7f7f7f || brk == INT_MAX ? -1 : brk;
  c->collect_kernel_stats();
  return c->stats.first_breakdown_col >= 0 ? RGSQR_WARN_RANK_DEFICIENT : RGSQR_OK;
}

}  // namespace rgsqr

// ------------------------------------------------------------------------------------
// NCCL (loaded at run time from the pip wheel torch uses; only for nranks > 1)
// ------------------------------------------------------------------------------------
namespace {
struct NcclApi {
  void* lib = nullptr;
  int (*getUniqueId)(void*) = nullptr;
  // ncclCommInitRank takes the 128-byte ncclUniqueId BY VALUE
  struct UniqueId {
    char internal[128];
  };
  int (*commInitRank)(void**, int, UniqueId, int) = nullptr;
  int (*commDestroy)(void*) = nullptr;
  int (*allReduce)(const void*, void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*allGather)(const void*, void*, size_t, int, void*, cudaStream_t) = nullptr;
  bool load() {
    if (lib) return true;
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char* nm : names) {
      lib = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
      if (lib) break;
    }
    if (!lib) return false;
    getUniqueId = reinterpret_cast<int (*)(void*)>(dlsym(lib, "ncclGetUniqueId"));
    commInitRank = reinterpret_cast<int (*)(void**, int, UniqueId, int)>(dlsym(lib, "ncclCommInitRank"));
    commDestroy = reinterpret_cast<int (*)(void*)>(dlsym(lib, "ncclCommDestroy"));
    allReduce = reinterpret_cast<int (*)(const void*, void*, size_t, int, int, void*, cudaStream_t)>(
        dlsym(lib, "ncclAllReduce"));
    allGather = reinterpret_cast<int (*)(const void*, void*, size_t, int, void*, cudaStream_t)>(
        dlsym(lib, "ncclAllGather"));
    return getUniqueId && commInitRank && commDestroy && allReduce && allGather;
  }
};
NcclApi g_nccl;

int create_impl(rgsqr_handle* h, int device) {
  if (!h) return RGSQR_ERR_INVALID_ARG;
  *h = nullptr;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return RGSQR_ERR_CUDA;
  if (device < 0 || device >= ndev) return RGSQR_ERR_INVALID_ARG;
  if (cudaSetDevice(device) != cudaSuccess) return RGSQR_ERR_CUDA;
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return RGSQR_ERR_CUDA;
  if (prop.major != 10) return RGSQR_ERR_UNSUPPORTED;  // sm_100a only
  Ctx* c = new (std::nothrow) Ctx();
  if (!c) return RGSQR_ERR_HOST_MEM;
  c->device = device;
  c->num_sms = prop.multiProcessorCount;
  if (cudaStreamCreateWithFlags(&c->st_own, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->st_h2d, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->st_d2h, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->st_d2r, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->st_h2d2, cudaStreamNonBlocking) != cudaSuccess ||
      cudaMalloc(&c->d_partials, sizeof(float) * 2 * (LEAF_MAX_W + 2) * 1024) != cudaSuccess ||
      cudaMalloc(&c->d_sn_partials, sizeof(float) * LEAF_MAX_G * 64 * 64) != cudaSuccess ||
      cudaMalloc(&c->d_shape, 64) != cudaSuccess ||
      cudaMalloc(&c->d_sn_r12op, 128 * 128 * 4) != cudaSuccess ||
      cudaMalloc(&c->d_counter, 4096) != cudaSuccess || cudaMalloc(&c->d_breakdown, 256) != cudaSuccess ||
      cudaMalloc(&c->d_xw, sizeof(unsigned long long) * LEAF_XW_WORDS * LEAF_XW_STRIDE) != cudaSuccess ||
      cudaMalloc(&c->d_xprev, sizeof(unsigned long long) * LEAF_XW_WORDS) != cudaSuccess ||
      cudaMalloc(&c->d_peers, sizeof(void*) * 64) != cudaSuccess ||
      cudaMalloc(&c->d_r0buf, sizeof(float) * (LEAF_MAX_W + 2)) != cudaSuccess ||
      cudaMemset(c->d_xw, 0, sizeof(unsigned long long) * LEAF_XW_WORDS * LEAF_XW_STRIDE) != cudaSuccess ||
      cudaMemset(c->d_xprev, 0, sizeof(unsigned long long) * LEAF_XW_WORDS) != cudaSuccess ||
      cudaMemset(c->d_counter, 0, 4096) != cudaSuccess ||
      cudaMemcpy(c->d_peers, &c->d_xw, sizeof(void*), cudaMemcpyHostToDevice) != cudaSuccess ||
      // (cudaMemset / pageable cudaMemcpy may return before the device write lands, and the work
      // streams are non-blocking: drain the device before any of them can read these buffers)
      cudaDeviceSynchronize() != cudaSuccess) {
    delete c;
    return RGSQR_ERR_CUDA;
  }
  // every context-lifetime device buffer counts against each call's device_mem_budget (the arena gets
  // the budget minus these bytes, stats.ctx_device_bytes)
  c->ctx_bytes = sizeof(float) * 2 * (LEAF_MAX_W + 2) * 1024 + sizeof(float) * LEAF_MAX_G * 64 * 64 + 128 * 128 * 4 +
                 4096 + 256 + sizeof(unsigned long long) * LEAF_XW_WORDS * LEAF_XW_STRIDE +
                 sizeof(unsigned long long) * LEAF_XW_WORDS + sizeof(void*) * 64 + sizeof(float) * (LEAF_MAX_W + 2) +
                 64;
  c->ctx_bytes = (c->ctx_bytes + 4095) / 4096 * 4096 + 10 * 512;   // (allocation granularity slack)
  reset_stats(c);
  *h = reinterpret_cast<rgsqr_handle>(c);
  return RGSQR_OK;
}

Ctx* C(rgsqr_handle h) { return reinterpret_cast<Ctx*>(h); }
}  // namespace

namespace rgsqr {
// Every rank of a row-sharded factorization must take identical planning decisions: check
// that the local row counts agree, use the smallest resolved budget, record the global m.
int sync_shape(Ctx* c, int64_t m, size_t* budget) {
  c->m_global = m;
  if (!c->nccl_comm) return RGSQR_OK;
  const size_t b = resolve_budget(c, *budget);
  int64_t h[3] = {m, -m, -(int64_t)b};
  int64_t* d = static_cast<int64_t*>(c->d_shape);   // (context buffer: no allocation per call)
  // stream-ordered: a pageable cudaMemcpy may return before its DMA lands, and the compute stream
  // is non-blocking -- the allreduce could then reduce (and we read back) the previous call's values
  cudaMemcpyAsync(d, h, sizeof(h), cudaMemcpyHostToDevice, c->compute());
  const int rc = g_nccl.allReduce(d, d, 3, NCCL_INT64, /*ncclMax*/ 2, c->nccl_comm, c->compute());
  cudaMemcpyAsync(h, d, sizeof(h), cudaMemcpyDeviceToHost, c->compute());
  cudaStreamSynchronize(c->compute());
  if (rc != 0) return fail(c, RGSQR_ERR_NCCL, "shape allreduce");
  if (h[0] != -h[1]) return fail(c, RGSQR_ERR_INVALID_ARG, "row-sharded run needs the same local m on every rank");
  *budget = (size_t)(-h[2]);
  c->m_global = m * c->nranks;
  return RGSQR_OK;
}

int nccl_allreduce(Ctx* c, void* buf, size_t count, int nccl_dtype, cudaStream_t st) {
  if (!c->nccl_comm) return RGSQR_OK;  // single-GPU context: nothing to reduce
  if (g_nccl.allReduce(buf, buf, count, nccl_dtype, /*ncclSum*/ 0, c->nccl_comm, st) != 0)
    return fail(c, RGSQR_ERR_NCCL, "ncclAllReduce failed");
  return RGSQR_OK;
}
}  // namespace rgsqr

extern "C" {

int rgsqr_version(void) { return 100; }

const char* rgsqr_status_string(int s) {
  switch (s) {
    case RGSQR_OK: return "RGSQR_OK";
    case RGSQR_WARN_RANK_DEFICIENT: return "RGSQR_WARN_RANK_DEFICIENT";
    case RGSQR_ERR_INVALID_ARG: return "RGSQR_ERR_INVALID_ARG";
    case RGSQR_ERR_BUDGET_TOO_SMALL: return "RGSQR_ERR_BUDGET_TOO_SMALL";
    case RGSQR_ERR_CUDA: return "RGSQR_ERR_CUDA";
    case RGSQR_ERR_NCCL: return "RGSQR_ERR_NCCL";
    case RGSQR_ERR_UNSUPPORTED: return "RGSQR_ERR_UNSUPPORTED";
    case RGSQR_ERR_HOST_MEM: return "RGSQR_ERR_HOST_MEM";
  }
  return "RGSQR_UNKNOWN_STATUS";
}

int rgsqr_create(rgsqr_handle* h, int device) { return create_impl(h, device); }

int rgsqr_get_unique_id(unsigned char id[128]) {
  if (!id) return RGSQR_ERR_INVALID_ARG;
  if (!g_nccl.load()) return RGSQR_ERR_NCCL;
  return g_nccl.getUniqueId(id) == 0 ? RGSQR_OK : RGSQR_ERR_NCCL;
}

static int create_dist_impl(Ctx* c, int rank, int nranks, const unsigned char id[128]);

int rgsqr_create_dist(rgsqr_handle* h, int device, int rank, int nranks, const unsigned char id[128]) {
  if (!h) return RGSQR_ERR_INVALID_ARG;
  *h = nullptr;
  if (nranks < 1 || rank < 0 || rank >= nranks || !id) return RGSQR_ERR_INVALID_ARG;
  if (nranks > 64) return RGSQR_ERR_UNSUPPORTED;
  int rc = create_impl(h, device);
  if (rc < 0) return rc;
  rc = create_dist_impl(C(*h), rank, nranks, id);
  if (rc < 0) {
    // release the streams, device buffers, IPC mappings and communicator created so far
    rgsqr_destroy(*h);
    *h = nullptr;
  }
  return rc;
}

static int create_dist_impl(Ctx* c, int rank, int nranks, const unsigned char id[128]) {
  c->rank = rank;
  c->nranks = nranks;
  // A distributed context always has an NCCL communicator (also for nranks == 1, which runs
  // the row-sharded code paths on one GPU: round-0 allreduce, R12 allreduce, .sys exchange).
  if (!g_nccl.load()) return fail(c, RGSQR_ERR_NCCL, "libnccl.so.2 not loadable");
  NcclApi::UniqueId uid;
  std::memcpy(uid.internal, id, sizeof(uid.internal));
  if (g_nccl.commInitRank(&c->nccl_comm, nranks, uid, rank) != 0) {
    c->nccl_comm = nullptr;
    return fail(c, RGSQR_ERR_NCCL, "ncclCommInitRank failed");
  }
  // Map every rank's leaf exchange words (CUDA IPC handles exchanged with ncclAllGather),
  // so the leaf kernel can red.add its partials into all GPUs' words over NVLink.
  std::vector<unsigned long long*> peers(nranks, nullptr);
  peers[rank] = c->d_xw;
  if (nranks > 1) {
    cudaIpcMemHandle_t mine;
    if (cudaIpcGetMemHandle(&mine, c->d_xw) != cudaSuccess) return fail(c, RGSQR_ERR_CUDA, "cudaIpcGetMemHandle");
    char* dbuf = nullptr;
    const size_t hs = sizeof(cudaIpcMemHandle_t);
    if (cudaMalloc(&dbuf, hs * (nranks + 1)) != cudaSuccess) return fail(c, RGSQR_ERR_CUDA, "cudaMalloc");
    cudaMemcpyAsync(dbuf + hs * nranks, &mine, hs, cudaMemcpyHostToDevice, c->st_own);
    if (g_nccl.allGather(dbuf + hs * nranks, dbuf, hs, /*ncclChar*/ 0, c->nccl_comm, c->st_own) != 0) {
      cudaFree(dbuf);
      return fail(c, RGSQR_ERR_NCCL, "ncclAllGather of IPC handles");
    }
    std::vector<cudaIpcMemHandle_t> all(nranks);
    cudaMemcpyAsync(all.data(), dbuf, hs * nranks, cudaMemcpyDeviceToHost, c->st_own);
    cudaStreamSynchronize(c->st_own);
    cudaFree(dbuf);
    for (int j = 0; j < nranks; ++j) {
      if (j == rank) continue;
      void* ptr = nullptr;
      if (cudaIpcOpenMemHandle(&ptr, all[j], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
        return fail(c, RGSQR_ERR_CUDA, "cudaIpcOpenMemHandle (peer " + std::to_string(j) + ")");
      peers[j] = static_cast<unsigned long long*>(ptr);
      c->ipc_opened.push_back(ptr);
    }
  }
  cudaMemcpyAsync(c->d_peers, peers.data(), sizeof(void*) * nranks, cudaMemcpyHostToDevice, c->st_own);
  // every rank has zeroed its words (create_impl) before anyone may add into them
  float one = 0.f;
  cudaMemcpyAsync(c->d_r0buf, &one, sizeof(float), cudaMemcpyHostToDevice, c->st_own);
  if (nccl_allreduce(c, c->d_r0buf, 1, NCCL_FLOAT32, c->st_own) < 0 || cudaStreamSynchronize(c->st_own) != cudaSuccess)
    return fail(c, RGSQR_ERR_NCCL, "initial barrier");
  return RGSQR_OK;
}

int rgsqr_destroy(rgsqr_handle h) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  cudaDeviceSynchronize();
  for (void* ptr : c->ipc_opened) cudaIpcCloseMemHandle(ptr);
  if (c->nccl_comm && g_nccl.commDestroy) g_nccl.commDestroy(c->nccl_comm);
  graph_drop_all(c);
  if (c->arena.base) cudaFree(c->arena.base);
  cudaFree(c->d_partials);
  cudaFree(c->d_sn_partials);
  cudaFree(c->d_sn_r12op);
  cudaFree(c->d_shape);
  cudaFree(c->d_counter);
  cudaFree(c->d_breakdown);
  cudaFree(c->d_xw);
  cudaFree(c->d_xprev);
  cudaFree(c->d_peers);
  cudaFree(c->d_r0buf);
  for (auto e : c->event_pool) cudaEventDestroy(e);
  for (auto& a : c->host_allocs) {
    cudaHostUnregister(a.first);
    munmap(a.first, a.second);
  }
  cudaStreamDestroy(c->st_own);
  cudaStreamDestroy(c->st_h2d);
  cudaStreamDestroy(c->st_d2h);
  cudaStreamDestroy(c->st_d2r);
  cudaStreamDestroy(c->st_h2d2);
  delete c;
  return RGSQR_OK;
}

int rgsqr_factor(rgsqr_handle h, const void* A_host, int64_t lda, int64_t m, int64_t n, void* Q_out, float* R_out,
                 int precision, size_t device_mem_budget) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  if (c->broken) return fail(c, RGSQR_ERR_CUDA, "handle unusable after a leaf exchange timeout: destroy it");
  return factor_host(c, A_host, lda, m, n, Q_out, R_out, precision, device_mem_budget);
}

int rgsqr_factor_device(rgsqr_handle h, const void* A_dev, int64_t lda, int64_t m, int64_t n, void* Q_dev,
                        float* R_dev, int precision, size_t device_mem_budget) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  if (c->broken) return fail(c, RGSQR_ERR_CUDA, "handle unusable after a leaf exchange timeout: destroy it");
  return factor_device(c, A_dev, lda, m, n, Q_dev, R_dev, precision, device_mem_budget);
}

int rgsqr_ooc_inner(rgsqr_handle h, const void* Q1_host, int64_t ldq, const void* A2_host, int64_t lda, int64_t m,
                    int64_t w1, int64_t w2, float* R12_host, int64_t ldr, int precision, int tiling, int64_t block,
                    size_t device_mem_budget) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  return ooc_gemm(c, 0, tiling, block, Q1_host, ldq, const_cast<void*>(A2_host), lda, R12_host, ldr, m, w1, w2,
                  precision, device_mem_budget);
}

int rgsqr_ooc_outer(rgsqr_handle h, const void* Q1_host, int64_t ldq, const float* R12_host, int64_t ldr,
                    void* A2_host, int64_t lda, int64_t m, int64_t w1, int64_t w2, int precision, int tiling,
                    int64_t block, size_t device_mem_budget) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  return ooc_gemm(c, 1, tiling, block, Q1_host, ldq, A2_host, lda, const_cast<float*>(R12_host), ldr, m, w1, w2,
                  precision, device_mem_budget);
}

int rgsqr_op_leaf(rgsqr_handle h, void* P, int64_t ldp, int64_t m, int64_t w, float* R11, int64_t ldr,
                  int precision, int* breakdown) {
  Ctx* c = C(h);
  if (!c || !P || !R11 || m < 1 || w < 1 || ldp < m || ldr < w) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  if (c->broken) return fail(c, RGSQR_ERR_CUDA, "handle unusable after a leaf exchange timeout: destroy it");
  cudaStream_t st = c->compute();
  RGSQR_CUDA(c, cudaMemsetAsync(c->d_breakdown, 0x7f, sizeof(int), st));
  int rc = op_leaf(c, precision, P, ldp, m, w, R11, ldr, 0, st);
  if (rc < 0) return rc;
  int brk = INT_MAX;
  RGSQR_CUDA(c, cudaMemcpyAsync(&brk, c->d_breakdown, sizeof(int), cudaMemcpyDeviceToHost, st));
  RGSQR_CUDA(c, cudaStreamSynchronize(st));
  if (brk == -2) {
    c->broken = true;
    return fail(c, RGSQR_ERR_CUDA, "leaf exchange timed out (a rank did not arrive)");
  }
  if (breakdown) *breakdown = (brk == 0x7f7f7f7f) ? -1 : brk;
  return brk == 0x7f7f7f7f ? RGSQR_OK : RGSQR_WARN_RANK_DEFICIENT;
}

int rgsqr_op_inner(rgsqr_handle h, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m, int64_t w1,
                   int64_t w2, float* R12, int64_t ldr, void* R12op, int accumulate, int precision) {
  Ctx* c = C(h);
  if (!c || !Q1 || !A2 || !R12 || m < 1 || w1 < 1 || w2 < 1 || ldr < w1) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  int rc = ensure_arena(c, (size_t)72 << 20);
  if (rc < 0) return rc;
  rc = op_inner(c, precision, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, R12op, w1, accumulate, c->compute());
  if (rc < 0) return rc;
  RGSQR_CUDA(c, cudaStreamSynchronize(c->compute()));
  return RGSQR_OK;
}

int rgsqr_op_outer(rgsqr_handle h, const void* Q1, int64_t ldq, const void* R12op, int64_t ldr, void* A2,
                   int64_t lda, int64_t m, int64_t w1, int64_t w2, int precision) {
  Ctx* c = C(h);
  if (!c || !Q1 || !A2 || !R12op || m < 1 || w1 < 1 || w2 < 1) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  int rc = op_outer(c, precision, Q1, ldq, R12op, ldr, A2, lda, m, w1, w2, c->compute());
  if (rc < 0) return rc;
  RGSQR_CUDA(c, cudaStreamSynchronize(c->compute()));
  return RGSQR_OK;
}

int rgsqr_set_stream(rgsqr_handle h, void* s) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  c->st_user = static_cast<cudaStream_t>(s);
  return RGSQR_OK;
}

int rgsqr_get_stream(rgsqr_handle h, void** s) {
  Ctx* c = C(h);
  if (!c || !s) return RGSQR_ERR_INVALID_ARG;
  *s = c->compute();
  return RGSQR_OK;
}

// NUMA node of the GPU (sysfs; -1 when unknown or single-node) and the CPUs of that node
static int gpu_numa_node(int device) {
  char bus[64] = {0};
  if (cudaDeviceGetPCIBusId(bus, sizeof(bus), device) != cudaSuccess) return -1;
  for (char* q = bus; *q; ++q) *q = (char)tolower(*q);
  std::string path = std::string("/sys/bus/pci/devices/") + bus + "/numa_node";
  FILE* f = fopen(path.c_str(), "r");
  if (!f) return -1;
  int node = -1;
  if (fscanf(f, "%d", &node) != 1) node = -1;
  fclose(f);
  return node;
}
static std::vector<int> node_cpus(int node) {
  std::vector<int> cpus;
  if (node < 0) return cpus;
  FILE* f = fopen(("/sys/devices/system/node/node" + std::to_string(node) + "/cpulist").c_str(), "r");
  if (!f) return cpus;
  char buf[4096] = {0};
  if (fgets(buf, sizeof(buf), f)) {
    for (char* tok = strtok(buf, ",\n"); tok; tok = strtok(nullptr, ",\n")) {
      int a = -1, b = -1;
      if (sscanf(tok, "%d-%d", &a, &b) == 2)
        for (int x = a; x <= b; ++x) cpus.push_back(x);
      else if (sscanf(tok, "%d", &a) == 1)
        cpus.push_back(a);
    }
  }
  fclose(f);
  return cpus;
}

// Pinned host memory placed on the GPU's NUMA node: anonymous pages first-touched by threads bound
// to that node's CPUs (the kernel's default policy allocates a page on the node of the CPU that first
// writes it), then page-locked for DMA with cudaHostRegister.  The touch runs on up to 16 threads.
int rgsqr_host_alloc(rgsqr_handle h, size_t bytes, void** p) {
  Ctx* c = C(h);
  if (!c || !p || bytes == 0) return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  void* mem = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (mem == MAP_FAILED) return fail(c, RGSQR_ERR_HOST_MEM, "mmap failed");
  const int node = gpu_numa_node(c->device);
  const std::vector<int> cpus = node_cpus(node);
  const int nt = (int)std::max<size_t>(1, std::min<size_t>(16, cpus.empty() ? 8 : cpus.size()));
  const size_t page = 4096, per = ((bytes + nt - 1) / nt + page - 1) / page * page;
  std::vector<std::thread> th;
  for (int t = 0; t < nt; ++t) {
    th.emplace_back([&, t] {
      if (!cpus.empty()) {
        cpu_set_t set;
        CPU_ZERO(&set);
        for (int cpu : cpus) CPU_SET(cpu, &set);
        pthread_setaffinity_np(pthread_self(), sizeof(set), &set);
      }
      const size_t a = std::min(bytes, (size_t)t * per), b = std::min(bytes, a + per);
      if (b > a) std::memset(static_cast<char*>(mem) + a, 0, b - a);
    });
  }
  for (auto& x : th) x.join();
  if (cudaHostRegister(mem, bytes, cudaHostRegisterPortable) != cudaSuccess) {
    cudaGetLastError();
    munmap(mem, bytes);
    return fail(c, RGSQR_ERR_HOST_MEM, "cudaHostRegister of the host buffer failed");
  }
  c->host_allocs[mem] = bytes;
  c->host_numa_node = node;
  *p = mem;
  return RGSQR_OK;
}

int rgsqr_host_free(rgsqr_handle h, void* p) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  auto it = c->host_allocs.find(p);
  if (it == c->host_allocs.end()) return fail(c, RGSQR_ERR_INVALID_ARG, "rgsqr_host_free: not from rgsqr_host_alloc");
  cudaHostUnregister(p);
  munmap(p, it->second);
  c->host_allocs.erase(it);
  return RGSQR_OK;
}

static int64_t* opt_slot(Ctx* c, int key) {
  Options& o = c->opt;
  switch (key) {
    case RGSQR_OPT_LEAF_WIDTH: return &o.leaf_width;
    case RGSQR_OPT_TILE_ROWS_MIN: return &o.tile_rows_min;
    case RGSQR_OPT_TILE_ROWS_MAX: return &o.tile_rows_max;
    case RGSQR_OPT_RING_DEPTH: return &o.ring_depth;
    case RGSQR_OPT_ALGO: return &o.algo;
    case RGSQR_OPT_BLOCK_COLS: return &o.block_cols;
    case RGSQR_OPT_SERIALIZE: return &o.serialize;
    case RGSQR_OPT_REUSE: return &o.reuse;
    case RGSQR_OPT_LEAF_CTAS: return &o.leaf_ctas;
    case RGSQR_OPT_SPLITK: return &o.splitk;
    case RGSQR_OPT_PROFILE: return &o.profile;
    case RGSQR_OPT_REORTH: return &o.reorth;
    case RGSQR_OPT_PREFETCH: return &o.prefetch;
    case RGSQR_OPT_FUSE_SMALL: return &o.fuse_small;
    case RGSQR_OPT_SPLIT_PCT: return &o.split_pct;
    case RGSQR_OPT_X3_CHAIN: return &o.x3_chain;
    case RGSQR_OPT_COLCHUNK: return &o.colchunk;
    case RGSQR_OPT_EAGER_PCT: return &o.eager_pct;
    case RGSQR_OPT_CHUNK_MIB: return &o.chunk_mib;
    case RGSQR_OPT_VSHARDS: return &o.vshards;
    case RGSQR_OPT_DEFER_PIECES: return &o.defer_pieces;
    case RGSQR_OPT_PHASEA_PCT: return &o.phasea_pct;
    case RGSQR_OPT_GRAPH: return &o.graph;
  }
  return nullptr;
}

int rgsqr_set_option(rgsqr_handle h, int key, int64_t value) {
  Ctx* c = C(h);
  if (!c) return RGSQR_ERR_INVALID_ARG;
  int64_t* s = opt_slot(c, key);
  if (!s) return fail(c, RGSQR_ERR_INVALID_ARG, "unknown option");
  switch (key) {
    case RGSQR_OPT_LEAF_WIDTH: if (value < 1 || value > LEAF_MAX_W) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_TILE_ROWS_MIN:
    case RGSQR_OPT_TILE_ROWS_MAX: if (value < 128 || value % 128) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_RING_DEPTH: if (value < 2 || value > 16) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_ALGO: if (value < 0 || value > 2) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_REORTH: if (value != 0 && value != 1) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_COLCHUNK:
    case RGSQR_OPT_GRAPH: if (value != 0 && value != 1) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_EAGER_PCT:
    case RGSQR_OPT_PHASEA_PCT: if (value < 0 || value > 100) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_CHUNK_MIB: if (value < 1 || value > 1024) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_VSHARDS: if (value < 1 || value > 64) return RGSQR_ERR_INVALID_ARG; break;
    case RGSQR_OPT_BLOCK_COLS: if (value < 8) return RGSQR_ERR_INVALID_ARG; break;
    default: if (value < 0) return RGSQR_ERR_INVALID_ARG;
  }
  *s = value;
  return RGSQR_OK;
}

int rgsqr_get_option(rgsqr_handle h, int key, int64_t* value) {
  Ctx* c = C(h);
  if (!c || !value) return RGSQR_ERR_INVALID_ARG;
  int64_t* s = opt_slot(c, key);
  if (!s) return RGSQR_ERR_INVALID_ARG;
  *value = *s;
  return RGSQR_OK;
}

int rgsqr_get_stats(rgsqr_handle h, rgsqr_stats* out) {
  Ctx* c = C(h);
  if (!c || !out) return RGSQR_ERR_INVALID_ARG;
  *out = c->stats;
  return RGSQR_OK;
}

int rgsqr_probe_link(rgsqr_handle h, void* host, int64_t ld, int64_t rows, int64_t cols, int elem_bytes, int reps,
                     double* gbps) {
  Ctx* c = C(h);
  if (!c || !host || !gbps || rows < 1 || cols < 1 || ld < rows || elem_bytes < 1 || reps < 1)
    return RGSQR_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  const size_t pitch = (size_t)ld * elem_bytes, wb = (size_t)rows * elem_bytes;
  const size_t tile = wb * cols;
  char* d = nullptr;
  RGSQR_CUDA(c, cudaMalloc(&d, 2 * tile));
  cudaEvent_t e[6];
  for (auto& x : e) cudaEventCreate(&x);
  auto up = [&](int r) { return cudaMemcpy2DAsync(d, wb, host, pitch, wb, cols, cudaMemcpyHostToDevice, c->st_h2d); };
  auto down = [&](int r) { return cudaMemcpy2DAsync(host, pitch, d + tile, wb, wb, cols, cudaMemcpyDeviceToHost, c->st_d2h); };
  cudaError_t err = cudaSuccess;
  // warm-up, then H2D alone, D2H alone, duplex (both streams, joined)
  err = up(0) == cudaSuccess && down(0) == cudaSuccess ? cudaSuccess : cudaErrorUnknown;
  cudaStreamSynchronize(c->st_h2d);
  cudaStreamSynchronize(c->st_d2h);
  cudaEventRecord(e[0], c->st_h2d);
  for (int r = 0; r < reps; ++r) up(r);
  cudaEventRecord(e[1], c->st_h2d);
  cudaStreamSynchronize(c->st_h2d);
  cudaEventRecord(e[2], c->st_d2h);
  for (int r = 0; r < reps; ++r) down(r);
  cudaEventRecord(e[3], c->st_d2h);
  cudaStreamSynchronize(c->st_d2h);
  cudaEventRecord(e[4], c->st_h2d);
  cudaStreamWaitEvent(c->st_d2h, e[4], 0);
  for (int r = 0; r < reps; ++r) {
    up(r);
    down(r);
  }
  cudaEvent_t j;
  cudaEventCreate(&j);
  cudaEventRecord(j, c->st_d2h);
  cudaStreamWaitEvent(c->st_h2d, j, 0);
  cudaEventRecord(e[5], c->st_h2d);
  cudaError_t e2 = cudaStreamSynchronize(c->st_h2d);
  float ms[3] = {0, 0, 0};
  cudaEventElapsedTime(&ms[0], e[0], e[1]);
  cudaEventElapsedTime(&ms[1], e[2], e[3]);
  cudaEventElapsedTime(&ms[2], e[4], e[5]);
  for (auto& x : e) cudaEventDestroy(x);
  cudaEventDestroy(j);
  cudaFree(d);
  if (err != cudaSuccess || e2 != cudaSuccess) return fail(c, RGSQR_ERR_CUDA, "probe_link copies failed");
  const double bytes = (double)tile * reps;
  gbps[0] = bytes / (ms[0] * 1e-3) / 1e9;
  gbps[1] = bytes / (ms[1] * 1e-3) / 1e9;
  gbps[2] = 2.0 * bytes / (ms[2] * 1e-3) / 1e9;
  return RGSQR_OK;
}

const char* rgsqr_last_error(rgsqr_handle h) {
  Ctx* c = C(h);
  if (!c) return "invalid handle";
  return c->last_error.c_str();
}

}  // extern "C"
