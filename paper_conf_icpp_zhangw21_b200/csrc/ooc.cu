// ooc.cu -- host-resident (out-of-core) recursive CGS QR: the executor.
//
// The recursion of Eq. (2) is walked on the host.  A node whose
// columns fit the device arena (the budget) is factored IN-CORE by the
// device recursion of ops.cu, its columns uploaded in chunks that the recursion waits
// on progressively, and its Q columns downloaded as soon as each leaf finishes
// (cross-operation overlap).  A node that does not fit is OUT-OF-CORE:
//
//   left child  -> inner product R12 = Q1^T A2, row tiles streamed (Fig. 3)
//               -> R12 out once at the end
//               -> outer product A2 <- A2 - Q1 R12, R12 resident, row tiles in and out
//                  (Fig. 5)
//   right child
//
// Row tiles move through a K-slot device ring on three streams (h2d copy engine,
// compute, d2h copy engine) chained by events: loaded[s] -> kernel -> done[s] -> d2h
// -> free[s] -> next upload into s.  Tile height ramps from tile_rows_min up to the
// slot size.  QR-level reuse, when it fits the budget:
//   rule 1: the left child's Q1 stays resident after its in-core factorization, so
//           both products stream only A2 tiles;
//   rule 3: each A2' tile is written over the rows of Q1 it no longer needs (after
//           Q1 was downloaded) instead of back to the host, so the right child starts
//           in-core without re-reading A2'  (the paper's "fast in-core data
//           transferring" D2D copy, used here to build the resident A2').
// The blocked algorithm (option ALGO=1) reuses the same node primitives
// with a fixed panel width instead of the recursion.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <chrono>
#include <climits>
#include <cstring>
#include <thread>
#include <vector>

#include "engine.h"

namespace rgsqr {
int ensure_arena(Ctx* c, size_t want);
size_t resolve_budget(Ctx* c, size_t budget);
void reset_stats(Ctx* c);
int validate(Ctx* c, const void* A, int64_t lda, int64_t m, int64_t n, const void* Q, int prec);

namespace {

struct Exec {
  Ctx* c;
  int prec;
  int64_t s;
  const char* A;
  char* Q;
  int64_t lda, m, n;
  float* R;
  cudaStream_t sc, sh, sd, sr;   // compute, h2d, Q d2h, R d2h
  int K;
  int64_t tmin, tmax;
  bool reuse;
  bool reorth;
  cudaStream_t sh2 = nullptr;    // second upload queue (column-chunked node's late tail piece)

  // ---- timing / accounting helpers ----
  // per-segment timing events; inside a graph capture only for RGSQR_TIMELINE, as external event
  // record nodes (events owned by the graph entry, valid after every replay)
  cudaEvent_t seg_event(cudaStream_t st) {
    cudaEvent_t e;
    if (c->capturing) {
      cudaEventCreate(&e);
      c->graph_tl_events.push_back(e);
      cudaEventRecordWithFlags(e, st, cudaEventRecordExternal);
    } else {
      e = c->ev();
      cudaEventRecord(e, st);
    }
    return e;
  }
  cudaEvent_t seg_begin(cudaStream_t st) {
    if (c->capturing && !c->graph_timeline) return nullptr;   // (replays are not timed per segment)
    return seg_event(st);
  }
  void seg_end(int kind, cudaStream_t st, cudaEvent_t a) {
    if (!a) return;
    cudaEvent_t b = seg_event(st);
    c->segs.push_back({kind, a, b});
  }
  void wait(cudaStream_t waiter, cudaStream_t signaller) {
    if (waiter == signaller) return;
    cudaEvent_t e = c->ev();
    cudaEventRecord(e, signaller);
    cudaStreamWaitEvent(waiter, e, 0);
  }
  // graph capture: the copy streams join the capture from the compute stream, and all of them
  // join back into it before the capture ends
  void fork_from_compute() {
    wait(sh, sc);
    wait(sd, sc);
    wait(sr, sc);
    if (sh2) wait(sh2, sc);
  }
  void join_into_compute() {
    wait(sc, sh);
    wait(sc, sd);
    wait(sc, sr);
    if (sh2) wait(sc, sh2);
  }
  void join_all() {
    wait(sc, sh);
    wait(sc, sd);
    wait(sc, sr);
    if (sh2) wait(sc, sh2);
    wait(sh, sc);
    wait(sd, sc);
    wait(sr, sc);
    if (sh2) wait(sh2, sc);
  }
  cudaEvent_t mark_ev(cudaStream_t st) {
    cudaEvent_t e = c->ev();
    cudaEventRecord(e, st);
    return e;
  }
  const char* hsrc(bool q) const { return q ? Q : A; }
  const char* hptr(const char* base, int64_t r0, int64_t col) const { return base + (r0 + col * lda) * s; }

  int h2d(void* dst, int64_t ldd, const char* base, int64_t r0, int64_t rows, int64_t c0, int64_t cols,
          cudaStream_t on = nullptr) {
    if (!on) on = sh;
    cudaEvent_t a = seg_begin(on);
    RGSQR_CUDA(c, cudaMemcpy2DAsync(dst, ldd * s, hptr(base, r0, c0), lda * s, rows * s, cols,
                                    cudaMemcpyHostToDevice, on));
    seg_end(0, on, a);
    c->stats.h2d_bytes += rows * cols * s;
    c->stats.h2d_matrix_bytes += rows * cols * s;
    return RGSQR_OK;
  }
  int d2h(char* base, int64_t r0, int64_t rows, int64_t c0, int64_t cols, const void* src, int64_t lds) {
    cudaEvent_t a = seg_begin(sd);
    RGSQR_CUDA(c, cudaMemcpy2DAsync(const_cast<char*>(hptr(base, r0, c0)), lda * s, src, lds * s, rows * s, cols,
                                    cudaMemcpyDeviceToHost, sd));
    seg_end(1, sd, a);
    c->stats.d2h_bytes += rows * cols * s;
    c->stats.d2h_matrix_bytes += rows * cols * s;
    return RGSQR_OK;
  }
  int d2h_r(int64_t r0, int64_t c0, int64_t rows, int64_t cols, const float* src, int64_t lds) {
    if (!R) return RGSQR_OK;  // non-zero ranks of a distributed run
    // R blocks go out on their own stream: they never queue behind a backlog of Q columns
    wait(sr, sc);
    cudaEvent_t a = seg_begin(sr);
    RGSQR_CUDA(c, cudaMemcpy2DAsync(R + r0 + c0 * n, n * sizeof(float), src, lds * sizeof(float),
                                    rows * sizeof(float), cols, cudaMemcpyDeviceToHost, sr));
    seg_end(1, sr, a);
    r_done = c->ev();
    cudaEventRecord(r_done, sr);
    c->stats.d2h_bytes += rows * cols * 4;
    c->stats.d2h_r_bytes += rows * cols * 4;
    return RGSQR_OK;
  }

  // ---- sizing ----
  size_t incore_need(int64_t w) const {
    return (size_t)m * w * s + 256 + (size_t)w * w * 4 + 256 + incore_workspace_bytes(c, prec, m, w) + 4096;
  }
  bool flat = false;   // no ramp: the first tiles were prefetched (see prefetch_tiles)
  cudaEvent_t r_done = nullptr;   // last R download issued
  std::vector<int64_t> tiles(int64_t t) const {
    std::vector<int64_t> v;
    int64_t r = 0, cur = flat ? t : std::min(tmin, t);
    while (r < m) {
      int64_t h = std::min(cur, m - r);
      v.push_back(h);
      r += h;
      cur = std::min(t, cur * 2);  // ramp
    }
    return v;
  }
  int64_t pick_tile(size_t avail, int64_t cols_per_slot, bool uncapped = false, int64_t w1w2 = 0) const {
    if (prec == RGSQR_TF32X3) {
      // leave room for the per-call hi/lo operands: 2 x (tile of Q1 + tile of A2) and the hi/lo
      // copies of R12 of the outer product
      const size_t r = (size_t)w1w2 * 8 + 4096;
      avail = avail > r ? (avail - r) / 3 : 0;
    }
    int64_t t = (int64_t)(avail / ((size_t)K * cols_per_slot * s));
    // the ramp's cap bounds streamed tiles; prefetched (flat) rings hold as
    // much of A2 as the budget allows
    if (!uncapped) t = std::min<int64_t>(t, tmax);
    t = std::min<int64_t>(t, (m + 127) / 128 * 128);
    t = t / 128 * 128;
    return t;
  }

  // ---- in-core node: upload (unless resident), factor, stream Q and R out ----
  // Rs_ext: caller-owned R block (kept alive by the caller, so no stream has to wait for
  // its download here); nullptr = allocate it from the arena and fence its reuse.
  // Feed of a node whose columns arrive from elsewhere (column-chunked OOC node, f4): uploads
  // already issued (column offset, completion event), one LATE chunk issued by the caller once
  // its memory is free (event filled in then), and a projection against an external Q1.
  struct Feed {
    std::vector<std::pair<int64_t, cudaEvent_t>> chunks;   // sorted by column; late one last
    int64_t late_col = -1;                                 // first column of the late chunk
    ExtProduct* ext = nullptr;
    int64_t eager_col = -1;   // leaf_done(col >= eager_col): apply the whole ext product now
    size_t next0 = 0;         // chunks before this index were already awaited by the compute stream
  };

  // defer_final (with Rs_ext): the last Q / R columns' download is returned as a closure instead of
  // issued, so that the caller can queue a more urgent copy ahead of it on the copy engine
  // defer_q_cols (with defer_final): the Q of the node's last defer_q_cols columns also waits for the
  // closure (the caller queues a more urgent copy ahead of it)
  int incore_node(int64_t c0, int64_t w, bool src_q, char* D, bool resident, cudaEvent_t* q_done,
                  float* Rs_ext = nullptr, Feed* feed = nullptr, std::function<int()>* defer_final = nullptr,
                  int64_t defer_q_cols = 0) {
    const size_t mark = c->arena.mark();
    float* Rs = Rs_ext ? Rs_ext : static_cast<float*>(c->arena.alloc((size_t)w * w * 4));
    if (!Rs) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "in-core node: no space for R block");
    RGSQR_CUDA(c, cudaMemsetAsync(Rs, 0, (size_t)w * w * 4, sc));
    const int64_t leaf = std::max(1, leaf_width_for(c, m));
    int64_t cw = (c->opt.chunk_mib << 20) / std::max<int64_t>(1, m * s);
    cw = std::max<int64_t>(leaf, cw / 64 * 64);
    std::vector<std::pair<int64_t, cudaEvent_t>> own;
    std::vector<std::pair<int64_t, cudaEvent_t>>& chunks = feed ? feed->chunks : own;
    if (!resident && !feed) {
      for (int64_t a = 0; a < w; a += cw) {
        const int64_t cols = std::min(cw, w - a);
        int rc = h2d(D + a * m * s, m, hsrc(src_q), 0, m, c0 + a, cols);
        if (rc < 0) return rc;
        cudaEvent_t e = c->ev();
        cudaEventRecord(e, sh);
        chunks.push_back({a, e});
      }
    }
    size_t next = feed ? feed->next0 : 0;
    int64_t flushed = 0;
    int err = 0;
    IncoreHooks hk;
    hk.need = [&](int64_t col_end) {
      while (next < chunks.size() && chunks[next].first < col_end) {
        if (!chunks[next].second) {   // a late chunk must be issued before anyone waits for it
          err = fail(c, RGSQR_ERR_CUDA, "column-chunked node: late chunk awaited before it was issued");
          return;
        }
        cudaStreamWaitEvent(sc, chunks[next].second, 0);
        ++next;
      }
    };
    // (a late chunk counts as pending only until it is issued: afterwards the recursion waits
    // for it instead of deferring whole products into column pieces)
    hk.pending = [&](int64_t col_end) {
      if (next >= chunks.size() || chunks[next].first >= col_end) return false;
      return !(feed && chunks[next].first == feed->late_col && chunks[next].second);
    };
    if (feed) hk.ext = feed->ext;
    // deferred products are applied in pieces of >= 256 columns (a multiple of the upload
    // chunk): narrower products (tall m makes cw small) would run at a fraction of the MMA rate
    hk.chunk = cw * std::max<int64_t>(1, (256 + cw - 1) / cw);
    // Q columns and the matching R columns (full height: entries below the diagonal are zero
    // and stay zero) go out as soon as a chunk of leaves is final
    hk.leaf_done = [&](int64_t col_end) {
      if (feed && feed->ext && feed->eager_col >= 0 && col_end >= feed->eager_col &&
          feed->ext->applied < feed->ext->end) {
        // apply the rest of the external projection now, so that Q1's memory frees (and the late
        // chunk uploads) while the recursion still works on earlier columns
        int rc = apply_ext(c, prec, D, m, m, &hk, feed->ext->end, sc);
        if (rc < 0) err = rc;
      }
      if (col_end - flushed < cw && col_end < w) return;
      wait(sd, sc);
      const int64_t qdefer = defer_final ? w - defer_q_cols : w;   // Q columns >= qdefer: in the closure
      int rc = flushed >= qdefer ? RGSQR_OK
                                 : d2h(Q, 0, m, c0 + flushed, std::min(col_end, qdefer) - flushed,
                                       D + flushed * m * s, m);
      // (rows [0, col_end) only: the rest of these columns is below the diagonal, zero, and the
      // host zeroes R_out's strict lower triangle itself)
      if (rc == 0) rc = d2h_r(c0, c0 + flushed, col_end, col_end - flushed, Rs + flushed * w, w);
      if (rc < 0) err = rc;
      flushed = col_end;
    };
    cudaEvent_t a = seg_begin(sc);
    int rc = incore_factor(c, prec, D, m, m, w, Rs, w, c0, sc, &hk);
    if (rc < 0) return rc;
    if (err < 0) return err;
    seg_end(2, sc, a);
    hk.need(w);  // (no-op unless the recursion skipped columns)
    wait(sd, sc);
    if (defer_final && Rs_ext) {
      cudaEvent_t ready = mark_ev(sc);
      const int64_t f0 = flushed, q0 = std::min(flushed, std::max<int64_t>(0, w - defer_q_cols));
      *defer_final = [this, ready, f0, q0, c0, w, D, Rs_ext]() -> int {
        cudaStreamWaitEvent(sd, ready, 0);
        if (f0 < w) {
          int r = d2h_r(c0, c0 + f0, w, w - f0, Rs_ext + f0 * w, w);
          if (r < 0) return r;
        }
        if (q0 < w) {
          int r = d2h(Q, 0, m, c0 + q0, w - q0, D + q0 * m * s, m);
          if (r < 0) return r;
        }
        return RGSQR_OK;
      };
      if (q_done) *q_done = nullptr;
      c->arena.release(mark);
      return RGSQR_OK;
    }
    if (flushed < w) {
      rc = d2h(Q, 0, m, c0 + flushed, w - flushed, D + flushed * m * s, m);
      if (rc < 0) return rc;
      rc = d2h_r(c0, c0 + flushed, w, w - flushed, Rs + flushed * w, w);
      if (rc < 0) return rc;
    }
    cudaEvent_t done = c->ev();
    cudaEventRecord(done, sd);
    if (q_done) *q_done = done;
    if (!Rs_ext && r_done) {
      // the R block lives in released arena space: nobody may reuse it before its download
      cudaStreamWaitEvent(sc, r_done, 0);
      cudaStreamWaitEvent(sh, r_done, 0);
    }
    c->arena.release(mark);
    return RGSQR_OK;
  }

  // ---- streamed inner product  R12 = Q1^T A2  (Q1 resident in D when D != null) ----
  int stream_inner(int64_t c0, int64_t w1, int64_t w2, bool a2_src_q, const char* D, float* R12, void* R12op,
                   char* ring, int64_t t, std::vector<cudaEvent_t>& ev_free,
                   const std::vector<cudaEvent_t>* pre = nullptr) {
    const int64_t h = c0 + w1;
    const int64_t slot_cols = (D ? 0 : w1) + w2;
    std::vector<cudaEvent_t> loaded(K);
    for (int k = 0; k < K; ++k) loaded[k] = c->ev();
    auto tl = tiles(t);
    int64_t r0 = 0;
    for (size_t i = 0; i < tl.size(); ++i) {
      const int64_t tr = tl[i];
      const int k = (int)(i % K);
      char* slot = ring + (size_t)k * t * slot_cols * s;
      char* sq = slot;
      char* sa = slot + (D ? 0 : (size_t)t * w1 * s);
      int rc;
      if (pre && i < pre->size()) {
        cudaStreamWaitEvent(sc, (*pre)[i], 0);            // uploaded during the left child
      } else {
        cudaStreamWaitEvent(sh, ev_free[k], 0);
        if (!D) {
          rc = h2d(sq, t, Q, r0, tr, c0, w1);
          if (rc < 0) return rc;
        }
        rc = h2d(sa, t, hsrc(a2_src_q), r0, tr, h, w2);
        if (rc < 0) return rc;
        cudaEventRecord(loaded[k], sh);
        cudaStreamWaitEvent(sc, loaded[k], 0);
      }
      cudaEvent_t a = seg_begin(sc);
      const bool last = (i + 1 == tl.size());
      // distributed: accumulate the LOCAL partial over all tiles, reduce across ranks once
      const bool dist = c->nccl_comm != nullptr;
      rc = op_inner(c, prec, D ? D + r0 * s : sq, D ? m : t, sa, t, tr, w1, w2, R12, w1,
                    (last && !dist) ? R12op : nullptr, w1, i > 0 ? 1 : 0, sc, /*reduce_ranks=*/false);
      if (rc < 0) return rc;
      if (last && dist) {
        rc = reduce_r12(c, prec, R12, w1, R12op, w1, w1, w2, sc);
        if (rc < 0) return rc;
      }
      seg_end(2, sc, a);
      cudaEventRecord(ev_free[k], sc);
      r0 += tr;
    }
    return RGSQR_OK;
  }

  // ---- cross-operation overlap: upload the first ring slots of the
  //      node's A2 while the left child is still being factored (the copy engine is idle
  //      once the left child's own columns are in); Q1 resident (rule 1) ----
  int prefetch_tiles(int64_t h, int64_t w2, bool a2_src_q, char* ring, int64_t t, std::vector<cudaEvent_t>* pre) {
    auto tl = tiles(t);
    int64_t r0 = 0;
    for (size_t i = 0; i < tl.size() && i < (size_t)K; ++i) {
      char* slot = ring + (size_t)i * t * w2 * s;
      int rc = h2d(slot, t, hsrc(a2_src_q), r0, tl[i], h, w2);
      if (rc < 0) return rc;
      cudaEvent_t e = c->ev();
      cudaEventRecord(e, sh);
      pre->push_back(e);
      r0 += tl[i];
    }
    return RGSQR_OK;
  }

  // ---- streamed outer product  A2 <- A2 - Q1 R12 ----
  // to_D: write A2' over Q1's rows in D (reuse rule 3) instead of downloading it.
  int stream_outer(int64_t c0, int64_t w1, int64_t w2, bool a2_src_q, char* D, bool to_D, cudaEvent_t q1_out_done,
                   const void* R12op, char* ring, int64_t t, std::vector<cudaEvent_t>& ev_free) {
    const int64_t h = c0 + w1;
    const int64_t slot_cols = (D ? 0 : w1) + w2;
    std::vector<cudaEvent_t> loaded(K), done(K);
    for (int k = 0; k < K; ++k) {
      loaded[k] = c->ev();
      done[k] = c->ev();
    }
    if (to_D && q1_out_done) cudaStreamWaitEvent(sc, q1_out_done, 0);
    auto tl = tiles(t);
    std::vector<int64_t> row0(tl.size());
    for (size_t i = 0, r = 0; i < tl.size(); r += tl[i], ++i) row0[i] = (int64_t)r;
    // Reuse: walk the tiles in REVERSE order, so the last K tiles of the
    // inner pass -- still in their ring slots, unmodified -- are consumed first without
    // being uploaded again.  Tile i always lives in slot i % K.
    const size_t n = tl.size();
    for (size_t j = 0; j < n; ++j) {
      const size_t i = reuse ? n - 1 - j : j;
      const int64_t tr = tl[i], r0 = row0[i];
      const int k = (int)(i % K);
      char* slot = ring + (size_t)k * t * slot_cols * s;
      char* sq = slot;
      char* sa = slot + (D ? 0 : (size_t)t * w1 * s);
      const bool resident = reuse && j < (size_t)K && i + K >= n;   // left in the slot by stream_inner
      if (!resident) {
        cudaStreamWaitEvent(sh, ev_free[k], 0);
        if (!D) {
          int rc = h2d(sq, t, Q, r0, tr, c0, w1);
          if (rc < 0) return rc;
        }
        int rc = h2d(sa, t, hsrc(a2_src_q), r0, tr, h, w2);
        if (rc < 0) return rc;
        cudaEventRecord(loaded[k], sh);
        cudaStreamWaitEvent(sc, loaded[k], 0);
      }
      int rc;
      cudaEvent_t a = seg_begin(sc);
      rc = op_outer(c, prec, D ? D + r0 * s : sq, D ? m : t, R12op, w1, sa, t, tr, w1, w2, sc);
      if (rc < 0) return rc;
      if (to_D) {
        RGSQR_CUDA(c, cudaMemcpy2DAsync(D + r0 * s, m * s, sa, t * s, tr * s, w2, cudaMemcpyDeviceToDevice, sc));
        c->stats.d2d_bytes += tr * w2 * s;
        seg_end(2, sc, a);
        cudaEventRecord(ev_free[k], sc);
      } else {
        seg_end(2, sc, a);
        cudaEventRecord(done[k], sc);
        cudaStreamWaitEvent(sd, done[k], 0);
        rc = d2h(Q, r0, tr, h, w2, sa, t);
        if (rc < 0) return rc;
        cudaEventRecord(ev_free[k], sd);
      }
    }
    return RGSQR_OK;
  }

  // ---- one out-of-core node: left, inner, outer, right ----
  // recursive = true: children are recursive nodes; false: blocked (left = panel,
  // right handled by the caller's loop).
  int ooc_node(int64_t c0, int64_t w1, int64_t w2, bool src_q, bool recursive) {
    c->stats.n_ooc_nodes++;
    const int64_t h = c0 + w1;
    const size_t mark0 = c->arena.mark();
    const size_t r12b = (size_t)w1 * w2 * 4 + 256, r12ob = (size_t)w1 * w2 * s + 256;
    // ---- reuse plan (rules 1 and 3) ----
    const size_t free0 = c->arena.free_bytes();
    const size_t dB = (size_t)m * w1 * s + 256;
    const size_t left_ws = incore_need(w1) - dB;
    const size_t right_ws = incore_need(w2) - (size_t)m * w2 * s;
    // the left child's R block + workspace and the node's R12 buffers are never live at the
    // same time: they share one scratch region above the ring (R12 is allocated there once
    // the left child's R block has been downloaded), so the ring can hold more of A2
    const size_t rsb = (size_t)w1 * w1 * 4;
    const size_t r12_all = r12b * (reorth ? 2 : 1) + r12ob;
    const size_t scratch = std::max(left_ws, r12_all + 1024) + 4096;   // left_ws includes the R block
    bool q1_res = reuse && dB + scratch + (size_t)K * 128 * w2 * s <= free0;
    bool a2_to_d = q1_res && recursive && w2 <= w1 && dB + right_ws <= free0;
    if (q1_res) {
      char* D = static_cast<char*>(c->arena.alloc(dB));
      const size_t avail = c->arena.free_bytes() > scratch ? c->arena.free_bytes() - scratch : 0;
      const int64_t t = D ? pick_tile(avail, w2, c->opt.prefetch != 0, w1 * w2) : 0;
      char* ring = t >= 128 ? static_cast<char*>(c->arena.alloc((size_t)K * t * w2 * s)) : nullptr;
      const size_t mark_s = c->arena.mark();
      float* Rs1 = ring ? static_cast<float*>(c->arena.alloc(rsb)) : nullptr;
      if (!D || !ring || !Rs1) {
        c->arena.release(mark0);
        q1_res = a2_to_d = false;
      } else {
        std::vector<cudaEvent_t> ev_free(K);
        for (int k = 0; k < K; ++k) ev_free[k] = c->ev();
        cudaEvent_t q1_done = nullptr;
        const bool saved_flat = flat;
        flat = c->opt.prefetch != 0;
        int rc = incore_node(c0, w1, src_q, D, false, &q1_done, Rs1);
        if (rc < 0) return rc;
        std::vector<cudaEvent_t> pre;
        if (flat) {
          rc = prefetch_tiles(h, w2, src_q, ring, t, &pre);
          if (rc < 0) return rc;
        }
        // the scratch region now holds R12: wait for the left child's R block download
        c->arena.release(mark_s);
        if (r_done) cudaStreamWaitEvent(sc, r_done, 0);
        float* R12 = static_cast<float*>(c->arena.alloc(r12b));
        void* R12op = c->arena.alloc(r12ob);
        float* S = reorth ? static_cast<float*>(c->arena.alloc(r12b)) : R12;
        if (!R12 || !R12op || !S) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "OOC node: no space for R12");
        rc = stream_inner(c0, w1, w2, src_q, D, R12, R12op, ring, t, ev_free, &pre);
        if (rc < 0) return rc;
        cudaEvent_t r12_out = nullptr;
        if (!reorth) {
          wait(sd, sc);
          rc = d2h_r(c0, h, w1, w2, R12, w1);
          if (rc < 0) return rc;
          r12_out = r_done;
        }
        rc = stream_outer(c0, w1, w2, src_q, D, a2_to_d && !reorth, q1_done, R12op, ring, t, ev_free);
        if (rc < 0) return rc;
        if (reorth) {
          // CGS2: S = Q1^T A2' (A2' from the host copy just written), R12 += S, A2' -= Q1 S
          rc = reorth_pass(c0, w1, w2, D, a2_to_d, q1_done, R12, S, R12op, ring, t, ev_free, &r12_out);
          if (rc < 0) return rc;
        }
        // R12 / ring memory is released below: make every stream wait for its last users
        if (r12_out) cudaStreamWaitEvent(sc, r12_out, 0);
        join_all();
        c->arena.release(mark0 + 0);
        flat = saved_flat;
        if (a2_to_d) {
          // keep D (now holding A2', rows permuted by nothing: same row order) for the right child
          char* D2 = static_cast<char*>(c->arena.alloc(dB));  // same address as D (LIFO)
          (void)D2;
          rc = incore_node(h, w2, true, D, true, nullptr);
          if (rc < 0) return rc;
          join_all();
          c->arena.release(mark0);
          return RGSQR_OK;
        }
        c->arena.release(mark0);
        return recursive ? node(h, w2, true) : RGSQR_OK;
      }
    }
    // ---- no reuse: Q1 tiles are re-read from the host ----
    int rc = recursive ? node(c0, w1, src_q) : panel(c0, w1, src_q);
    if (rc < 0) return rc;
    join_all();
    float* R12 = static_cast<float*>(c->arena.alloc(r12b));
    void* R12op = c->arena.alloc(r12ob);
    float* S = reorth ? static_cast<float*>(c->arena.alloc(r12b)) : R12;
    if (!R12 || !R12op || !S) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "OOC node: no space for R12");
    const int64_t t = pick_tile(c->arena.free_bytes() > 4096 ? c->arena.free_bytes() - 4096 : 0, w1 + w2, false, w1 * w2);
    if (t < 128) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "OOC node: ring does not fit the budget");
    char* ring = static_cast<char*>(c->arena.alloc((size_t)K * t * (w1 + w2) * s));
    std::vector<cudaEvent_t> ev_free(K);
    for (int k = 0; k < K; ++k) ev_free[k] = c->ev();
    rc = stream_inner(c0, w1, w2, src_q, nullptr, R12, R12op, ring, t, ev_free);
    if (rc < 0) return rc;
    if (!reorth) {
      wait(sd, sc);
      rc = d2h_r(c0, h, w1, w2, R12, w1);
      if (rc < 0) return rc;
    }
    rc = stream_outer(c0, w1, w2, src_q, nullptr, false, nullptr, R12op, ring, t, ev_free);
    if (rc < 0) return rc;
    if (reorth) {
      rc = reorth_pass(c0, w1, w2, nullptr, false, nullptr, R12, S, R12op, ring, t, ev_free, nullptr);
      if (rc < 0) return rc;
    }
    join_all();
    c->arena.release(mark0);
    return recursive ? node(h, w2, true) : RGSQR_OK;
  }

  // CGS2 second projection of an OOC node: A2' lives in the host Q copy (written by the
  // first outer pass).  S = Q1^T A2', R12 += S (then R12 is written out once), A2'' =
  // A2' - Q1 S (to D when to_D: Q1 is no longer needed after this pass).
  int reorth_pass(int64_t c0, int64_t w1, int64_t w2, char* D, bool to_D, cudaEvent_t q1_done, float* R12,
                  float* S, void* Sop, char* ring, int64_t t, std::vector<cudaEvent_t>& ev_free,
                  cudaEvent_t* r12_out) {
    const int64_t h = c0 + w1;
    int rc = stream_inner(c0, w1, w2, true, D, S, Sop, ring, t, ev_free);
    if (rc < 0) return rc;
    cudaEvent_t a = seg_begin(sc);
    switch (prec) {
      case RGSQR_FP16:
        RGSQR_CUDA(c, launch_splitk_reduce<__half>(S, w1 * w2, w1, 1, R12, w1, 1, nullptr, 0, w1, w2, sc));
        break;
      case RGSQR_BF16:
        RGSQR_CUDA(c, launch_splitk_reduce<__nv_bfloat16>(S, w1 * w2, w1, 1, R12, w1, 1, nullptr, 0, w1, w2, sc));
        break;
      default:
        RGSQR_CUDA(c, launch_splitk_reduce<float>(S, w1 * w2, w1, 1, R12, w1, 1, nullptr, 0, w1, w2, sc));
    }
    c->stats.n_other_launches++;
    seg_end(2, sc, a);
    wait(sd, sc);
    rc = d2h_r(c0, h, w1, w2, R12, w1);
    if (rc < 0) return rc;
    if (r12_out) {
      *r12_out = r_done;
    }
    return stream_outer(c0, w1, w2, true, D, to_D, q1_done, Sop, ring, t, ev_free);
  }

  int panel(int64_t c0, int64_t w, bool src_q) {
    const size_t mark = c->arena.mark();
    char* D = static_cast<char*>(c->arena.alloc((size_t)m * w * s));
    if (!D || c->arena.free_bytes() + 0 < incore_need(w) - (size_t)m * w * s)
      return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "panel of " + std::to_string(w) + " columns does not fit");
    int rc = incore_node(c0, w, src_q, D, false, nullptr);
    if (rc < 0) return rc;
    join_all();
    c->arena.release(mark);
    return RGSQR_OK;
  }

  // ---- column-chunked out-of-core node (f4, R26) ----------------------------------
  // The left child fits in-core: Q1 stays resident (rule 1).  A2 is split by COLUMNS into a head
  // [0, wh) that fits beside Q1 and a tail [wh, w2) that does not.  Arena layout:
  //     [ H : m x wh  (head; its top part first hosts the left child's workspace) ]
  //     [ D : m x w1  (Q1; after Q1 is dead its first wt columns receive the tail) ]
  //     [ X :         (tail piece T1 while prefetched, then the right child's workspace) ]
  // so that [H | D[:, :wt]] is the right child's contiguous m x w2 matrix (ld m).
  //   1. left child in-core in D (its columns uploaded in chunks, Q1 downloaded as leaves end);
  //      uploads queue behind it: the tail piece T1 (into X), then the head columns (into H).
  //   2. tail: R12_t = Q1^T A2_t, A2_t -= Q1 R12_t (Eq. 2) on the resident tail
  //      pieces, R12_t and A2_t' downloaded (A2_t' parked in the host Q columns it will occupy).
  //   3. right child in-core on [H | D[:, :wt]] at once: the head's R12 = Q1^T A2 and
  //      A2 -= Q1 R12 are applied column chunk by column chunk as the recursion reaches the
  //      columns (ExtProduct, ancestor first), completed eagerly part-way through; then Q1 is
  //      dead and A2_t' is uploaded into D while the recursion continues on earlier columns.
  // Same arithmetic per output element as the streamed node: every R12 column is Q1^T a_j over
  // all m rows and every A2' column is a_j - Q1 r_j (the column split only regroups the GEMMs).
  struct CCPlan {
    int64_t wh = 0, wt1 = 0, wt2 = 0;
    size_t htop = 0;                 // bytes at the top of H used as scratch (left child, tail phase)
    int64_t ch = 0;                  // upload / product chunk width
    int64_t E1 = 0;                  // head columns projected before the right child (phase A)
    int64_t pA = 0;                  // phase-A piece width
    int64_t pB = 0;                  // piece width of the remaining projection (phase B)
  };
  bool plan_cc(int64_t w1, int64_t w2, size_t free0, CCPlan* P) const {
    if ((m * s * 64) % 256 != 0) return false;   // (the tail must fit D: wt <= w1, checked below)
    const int64_t leaf = std::max(1, leaf_width_for(c, m));
    int64_t cw = (c->opt.chunk_mib << 20) / std::max<int64_t>(1, m * s);
    cw = std::max<int64_t>(leaf, cw / 64 * 64);
    const int64_t ch = cw * std::max<int64_t>(1, (256 + cw - 1) / cw);
    const size_t colb = (size_t)m * s, dB = (size_t)m * w1 * s;
    const size_t left_ws = incore_need(w1) - dB + 4096;
    const int64_t hw = split_width(w2, leaf);
    const int64_t pB = std::min<int64_t>(w2, 2 * ch);                 // phase-B piece (in X)
    const size_t ext_b = (size_t)w1 * pB * (4 + s) + 512;
    const size_t right_ws = (size_t)w2 * w2 * 4 + 256 + incore_workspace_bytes(c, prec, m, w2) + ext_b + 16384;
    const size_t rs1 = ((size_t)w1 * w1 * 4 + 255) / 256 * 256;
    for (int64_t wh = (w2 - 1) / 64 * 64; wh >= std::max<int64_t>(64, w2 / 4); wh -= 64) {
      const size_t H = colb * wh;
      if (H + dB + right_ws > free0) continue;
      const int64_t wt = w2 - wh;
      const size_t X = free0 - H - dB;
      const int64_t wt1 = std::min<int64_t>(wt, (int64_t)(X / colb) / 8 * 8);
      const int64_t wt2 = wt - wt1;
      const size_t tail_ws = (size_t)w1 * wt * (4 + s) + 1024 + (size_t)wt2 * colb + 256;
      // phase A: the right child's first half of head columns (E1) projected before it starts, in
      // pieces of pA columns (two fp32 R12 buffers + one operand buffer), while the tail goes out
      const int64_t E1 = std::min<int64_t>(wh, (hw * c->opt.phasea_pct / 100) / ch * ch);
      const int64_t pA = std::max<int64_t>(ch, std::min<int64_t>(E1, 2 * ch));
      const size_t phaseA = (size_t)w1 * pA * (8 + s) + 1024;
      const size_t t2 = (size_t)wt2 * colb + 256;
      const size_t htop = (std::max({left_ws, rs1 + tail_ws, rs1 + t2 + phaseA}) + 4095) / 4096 * 4096;
      if (htop > H || wt > w1) continue;
      P->wh = wh;
      P->wt1 = wt1;
      P->wt2 = wt2;
      P->htop = htop;
      P->ch = ch;
      P->E1 = E1;
      P->pA = pA;
      P->pB = pB;
      return true;
    }
    return false;
  }

  // sets the arena's bump window to [lo, hi) (allocations of a phase that lives inside a region
  // reserved by an earlier allocation); returns the previous (top, size)
  std::pair<size_t, size_t> window(char* lo, char* hi) {
    std::pair<size_t, size_t> w{c->arena.top, c->arena.size};
    c->arena.top = (size_t)(lo - c->arena.base);
    c->arena.size = (size_t)(hi - c->arena.base);
    return w;
  }
  void unwindow(std::pair<size_t, size_t> w) {
    c->arena.top = w.first;
    c->arena.size = w.second;
  }

  int ooc_node_cc(int64_t c0, int64_t w1, int64_t w2, bool src_q, const CCPlan& P) {
    const int64_t h = c0 + w1, wh = P.wh, wt1 = P.wt1, wt2 = P.wt2, wt = wt1 + wt2, ch = P.ch;
    const size_t colb = (size_t)m * s;
    const size_t mark0 = c->arena.mark();
    char* H = static_cast<char*>(c->arena.alloc(colb * wh));
    char* D = static_cast<char*>(c->arena.alloc(colb * w1));
    if (!H || !D || D != H + colb * wh) {
      c->arena.release(mark0);
      return 1;   // layout not contiguous: caller falls back to the streamed node
    }
    c->stats.n_ooc_nodes++;
    c->stats.n_colchunk_nodes++;
    c->stats.colchunk_tail_cols += wt;
    char* T1 = wt1 > 0 ? static_cast<char*>(c->arena.alloc(colb * wt1)) : nullptr;
    if (wt1 > 0 && !T1) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "column-chunked node: no space for the tail");
    const size_t x_mark = c->arena.mark();   // (X holds T1 until the right child starts)
    char* Hend = H + colb * wh;
    char* Htop = Hend - P.htop;
    const int64_t htop_col = (int64_t)((size_t)(Htop - H) / colb);   // head columns clear of the scratch
    // ---- 1. left child in-core in D; its workspace lives in the top of H ----
    auto wsave = window(Htop, Hend);
    float* Rs1 = static_cast<float*>(c->arena.alloc((size_t)w1 * w1 * 4));
    if (!Rs1) {
      unwindow(wsave);
      return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "column-chunked node: no space for the left R block");
    }
    cudaEvent_t q1_done = nullptr;
    std::function<int()> left_final;   // the left child's last Q / R download, queued after the tail's
    // (RGSQR_DEFER_Q_CHUNKS > 0: the Q of its last few upload chunks too, queued behind the tail's
    // download -- measured slower at configs[1]: 37.6 / 37.9 / 38.6 ms for 3 / 4 / 6 chunks vs 37.1)
    static const int64_t dq_env = getenv("RGSQR_DEFER_Q_CHUNKS") ? atoll(getenv("RGSQR_DEFER_Q_CHUNKS")) : 0;
    int rc = incore_node(c0, w1, src_q, D, false, &q1_done, Rs1, nullptr, &left_final, dq_env * ch);
    unwindow(wsave);
    if (rc < 0) return rc;
    cudaEvent_t left_done = mark_ev(sc);
    // ---- uploads queued behind the left child's: tail piece 1, then the head clear of H's top ----
    cudaEvent_t ev_t1 = nullptr, ev_t2 = nullptr;
    if (wt1 > 0) {
      rc = h2d(T1, m, hsrc(src_q), 0, m, h + wh, wt1);
      if (rc < 0) return rc;
      ev_t1 = mark_ev(sh);
    }
    // head chunks clear of H's top; the tail's second piece goes in after the first two (it waits for
    // the left child, and a copy queued behind the whole head would arrive long after it is needed:
    // uploads from all streams share the copy engine in submission order)
    Feed feed;
    auto head_chunk = [&](int64_t a, int64_t end) -> int {
      int r = h2d(H + a * colb, m, hsrc(src_q), 0, m, h + a, end - a);
      if (r < 0) return r;
      feed.chunks.push_back({a, mark_ev(sh)});
      return RGSQR_OK;
    };
    // ---- 2. the tail: workspace and second piece in the top of H, above the left R block (so that
    //      nothing waits for that block's download) ----
    // (T2 first: phase A's buffers later go above T2 -- T2 is downloaded while phase A runs -- and over
    // the tail's R12 buffers, whose use is over by then)
    const size_t rs1b = ((size_t)w1 * w1 * 4 + 255) / 256 * 256;
    wsave = window(Htop + rs1b, Hend);
    char* T2 = wt2 > 0 ? static_cast<char*>(c->arena.alloc(colb * wt2)) : nullptr;
    float* R12t = static_cast<float*>(c->arena.alloc((size_t)w1 * wt * 4));
    char* R12top = static_cast<char*>(c->arena.alloc((size_t)w1 * wt * s));
    unwindow(wsave);
    const size_t t2b = wt2 > 0 ? (colb * wt2 + 255) / 256 * 256 : 0;
    if (!R12t || !R12top || (wt2 > 0 && !T2))
      return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "column-chunked node: no space for the tail products");
    int64_t a_head = 0;
    for (int k = 0; k < 2 && a_head < htop_col; ++k) {
      const int64_t e = std::min(htop_col, a_head + ch);
      if ((rc = head_chunk(a_head, e)) < 0) return rc;
      a_head = e;
    }
    if (wt2 > 0) {
      cudaStreamWaitEvent(sh, left_done, 0);
      rc = h2d(T2, m, hsrc(src_q), 0, m, h + wh + wt1, wt2);
      if (rc < 0) return rc;
      ev_t2 = mark_ev(sh);
    }
    for (; a_head < htop_col;) {
      const int64_t e = std::min(htop_col, a_head + ch);
      if ((rc = head_chunk(a_head, e)) < 0) return rc;
      a_head = e;
    }
    cudaEvent_t a_seg = seg_begin(sc);
    struct Piece { char* T; int64_t col, w; cudaEvent_t ev; };
    const Piece pieces[2] = {{T1, 0, wt1, ev_t1}, {T2, wt1, wt2, ev_t2}};
    for (const Piece& pc : pieces) {
      if (pc.w == 0) continue;
      cudaStreamWaitEvent(sc, pc.ev, 0);
      rc = op_inner(c, prec, D, m, pc.T, m, m, w1, pc.w, R12t + pc.col * w1, w1, R12top + pc.col * w1 * s, w1, 0, sc);
      if (rc < 0) return rc;
    }
    rc = d2h_r(c0, h + wh, w1, wt, R12t, w1);
    if (rc < 0) return rc;
    cudaEvent_t r12t_out = r_done;
    for (const Piece& pc : pieces) {
      if (pc.w == 0) continue;
      rc = op_outer(c, prec, D, m, R12top + pc.col * w1 * s, w1, pc.T, m, m, w1, pc.w, sc);
      if (rc < 0) return rc;
    }
    wait(sd, sc);
    for (const Piece& pc : pieces) {
      if (pc.w == 0) continue;
      rc = d2h(Q, 0, m, h + wh + pc.col, pc.w, pc.T, m);   // A2_t' parked in its host Q columns
      if (rc < 0) return rc;
    }
    cudaEvent_t tail_out = mark_ev(sd);
    // now the left child's last columns (nothing waits on them but the end of the call and the reuse of
    // H's top, which holds its R block)
    if (left_final && (rc = left_final()) < 0) return rc;
    cudaEvent_t left_r = r_done;
    cudaEvent_t left_q = mark_ev(sd);
    // ---- phase A: the first E1 head columns' projection in one piece (buffers at the bottom of H's
    //      top, once the left R block is downloaded), while the tail goes out ----
    ExtProduct ext;
    ext.Q1 = D;
    ext.ldq = m;
    ext.w1 = w1;
    ext.end = wh;
    ext.r_out = [&](int64_t a, int64_t b, const float* R12) -> cudaEvent_t {
      if (d2h_r(c0, h + a, w1, b - a, R12, w1) < 0) return nullptr;
      return r_done;
    };
    size_t waited = 0;
    IncoreHooks hkA;
    hkA.chunk = ch;
    hkA.ext = &ext;
    hkA.need = [&](int64_t col_end) {
      while (waited < feed.chunks.size() && feed.chunks[waited].first < col_end)
        cudaStreamWaitEvent(sc, feed.chunks[waited++].second, 0);
    };
    const int64_t E1 = std::min<int64_t>(P.E1, htop_col / ch * ch);   // (its columns must be uploaded)
    cudaEvent_t phaseA_r[2] = {nullptr, nullptr};
    if (E1 > 0) {
      const int64_t pA = std::min<int64_t>(P.pA, E1);
      // (above the left R block and T2, both still downloading; over the tail's R12, which must be out)
      if (r12t_out) cudaStreamWaitEvent(sc, r12t_out, 0);
      wsave = window(Htop + rs1b + t2b, Hend);
      ext.R12[0] = static_cast<float*>(c->arena.alloc((size_t)w1 * pA * 4));
      ext.R12[1] = static_cast<float*>(c->arena.alloc((size_t)w1 * pA * 4));
      ext.R12op = c->arena.alloc((size_t)w1 * pA * s);
      unwindow(wsave);
      if (!ext.R12[0] || !ext.R12[1] || !ext.R12op)
        return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "column-chunked node: no space for the first projection");
      ext.piece = pA;
      rc = apply_ext(c, prec, H, m, m, &hkA, E1, sc);
      if (rc < 0) return rc;
      phaseA_r[0] = ext.free_ev[0];
      phaseA_r[1] = ext.free_ev[1];
    }
    seg_end(2, sc, a_seg);
    cudaEvent_t phaseA_done = mark_ev(sc);
    // the rest of the head goes into H's top once the tail phase and phase A have released it
    cudaStreamWaitEvent(sh, phaseA_done, 0);
    cudaStreamWaitEvent(sh, tail_out, 0);
    if (left_r) cudaStreamWaitEvent(sh, left_r, 0);   // (H's top held the left R block)
    if (r12t_out) cudaStreamWaitEvent(sh, r12t_out, 0);
    for (cudaEvent_t e : phaseA_r)
      if (e) cudaStreamWaitEvent(sh, e, 0);
    for (int64_t a = htop_col; a < wh;) {
      const int64_t end = std::min(wh, (a / ch + 1) * ch);
      if ((rc = head_chunk(a, end)) < 0) return rc;
      a = end;
    }
    // ---- 3. the right child, with the rest of the head's projection applied as its columns are
    //      reached and completed eagerly part-way through ----
    cudaStreamWaitEvent(sc, tail_out, 0);          // X (T1) becomes the right child's workspace
    c->arena.release(T1 ? (size_t)(T1 - c->arena.base) : x_mark);
    ext.piece = P.pB;
    ext.R12[0] = static_cast<float*>(c->arena.alloc((size_t)w1 * P.pB * 4));
    ext.R12[1] = nullptr;
    ext.R12op = c->arena.alloc((size_t)w1 * P.pB * s);
    ext.free_ev[0] = ext.free_ev[1] = nullptr;
    if (!ext.R12[0] || !ext.R12op)
      return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "column-chunked node: no space for the projection pieces");
    feed.late_col = wh;
    feed.chunks.push_back({wh, nullptr});
    feed.next0 = waited;
    ext.done = [&]() {
      // Q1 is dead once the compute stream gets here: the tail goes into D's first columns
      cudaEvent_t q1_dead = mark_ev(sc);
      cudaStreamWaitEvent(sh, q1_dead, 0);
      cudaStreamWaitEvent(sh, tail_out, 0);
      cudaStreamWaitEvent(sh, left_q, 0);   // (Q1's deferred last columns are on the host)
      if (h2d(D, m, Q, 0, m, h + wh, wt) < 0) return;
      feed.chunks.back().second = mark_ev(sh);
    };
    feed.ext = &ext;
    const int64_t leaf = std::max(1, leaf_width_for(c, m));
    const int64_t hw = split_width(w2, leaf);
    feed.eager_col = hw > 0 ? std::max<int64_t>(leaf, hw * c->opt.eager_pct / 100) : -1;
    rc = incore_node(h, w2, true, H, true, nullptr, nullptr, &feed);
    if (rc < 0) return rc;
    if (ext.applied < ext.end) return fail(c, RGSQR_ERR_CUDA, "column-chunked node: projection incomplete");
    join_all();
    c->arena.release(mark0);
    return RGSQR_OK;
  }

  // recursive algorithm (Eq. 2)
  int node(int64_t c0, int64_t w, bool src_q) {
    if (incore_need(w) <= c->arena.free_bytes()) return panel(c0, w, src_q);
    int64_t w1 = split_width(w, std::max(1, leaf_width_for(c, m)));
    if (w1 == 0) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "budget cannot hold one leaf panel");
    if (c->opt.split_pct != 50 && w >= 256) {
      // ablation (RGSQR_OPT_SPLIT_PCT): a larger left child, factored while the host link is
      // busy anyway, leaves a shorter right child -- the one phase that cannot overlap transfers
      const int64_t t = (w * c->opt.split_pct / 100 + 63) / 64 * 64;
      if (t >= 64 && t <= w - 64) w1 = t;
    }
    CCPlan P;
    if (c->opt.colchunk && reuse && !reorth && prec != RGSQR_TF32X3 && sh2 != nullptr &&
        plan_cc(w1, w - w1, c->arena.free_bytes(), &P)) {
      int rc = ooc_node_cc(c0, w1, w - w1, src_q, P);
      if (rc != 1) return rc;
    }
    return ooc_node(c0, w1, w - w1, src_q, true);
  }

  // blocked algorithm: panels of width b, trailing update streamed
  int blocked(int64_t b) {
    for (int64_t c0 = 0; c0 < n; c0 += b) {
      const int64_t w1 = std::min(b, n - c0), w2 = n - c0 - w1;
      int rc = (w2 == 0) ? panel(c0, w1, c0 > 0) : ooc_node(c0, w1, w2, c0 > 0, false);
      if (rc < 0) return rc;
    }
    return RGSQR_OK;
  }

  // fused blocked algorithm (RGSQR_OPT_ALGO = 2; SURVEY.md 8(f) f1 "honesty" variant and f4's
  // "fused-blocked top level"): the blocked loop of PAPER.md:113, but the panel Q stays resident and
  // the trailing matrix streams through in COLUMN blocks, each read once and written once per panel:
  // R12_j = Q^T A2_j and A2_j -= Q R12_j on the block while it is on the device (Fig. 4's inner tiling
  // fused with the outer update).  Per panel i the trailing (n - ib) columns move once each way, so the
  // whole factorization moves ~ (k+1)/2 m n words each way for k panels.
  int fused_blocked(int64_t b) {
    for (int64_t c0 = 0; c0 < n; c0 += b) {
      const int64_t w1 = std::min(b, n - c0), rest = n - c0 - w1;
      const bool src_q = c0 > 0;   // after the first panel the working matrix is the host Q copy
      const size_t mark = c->arena.mark();
      char* D = static_cast<char*>(c->arena.alloc((size_t)m * w1 * s));
      if (!D || c->arena.free_bytes() < incore_need(w1) - (size_t)m * w1 * s)
        return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "fused blocked: panel of " + std::to_string(w1) + " columns does not fit");
      cudaEvent_t q_done = nullptr;
      int rc = incore_node(c0, w1, src_q, D, false, &q_done);
      if (rc < 0) return rc;
      if (rest > 0) {
        c->stats.n_ooc_nodes++;
        // K column-block slots: A2 block (m x cb), its R12 (fp32) and operand copy
        const size_t per_col = (size_t)m * s + (size_t)w1 * (4 + s);
        const size_t fr = c->arena.free_bytes();
        const size_t ws = std::min<size_t>((size_t)16 << 20, fr / 4);   // split-K partials of the block products
        int64_t cb = fr > ws ? (int64_t)((fr - ws) / ((size_t)K * per_col)) : 0;
        cb = std::min<int64_t>(cb, rest);
        if (cb >= 64) cb = cb / 64 * 64;
        if (cb < 8) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "fused blocked: no room for column blocks");
        const size_t slot_b = ((size_t)m * cb * s + 255) / 256 * 256, rb = ((size_t)w1 * cb * 4 + 255) / 256 * 256;
        char* ring = static_cast<char*>(c->arena.alloc((size_t)K * (slot_b + rb + (size_t)w1 * cb * s + 256)));
        if (!ring) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "fused blocked: ring");
        std::vector<cudaEvent_t> freed(K, nullptr);
        const int64_t h = c0 + w1;
        int64_t j = 0;
        for (int64_t a = 0; a < rest; a += cb, ++j) {
          const int64_t cw = std::min(cb, rest - a);
          const int k = (int)(j % K);
          char* sa = ring + (size_t)k * (slot_b + rb + (size_t)w1 * cb * s + 256);
          float* sr = reinterpret_cast<float*>(sa + slot_b);
          char* so = sa + slot_b + rb;
          if (freed[k]) {
            cudaStreamWaitEvent(sh, freed[k], 0);
            cudaStreamWaitEvent(sc, freed[k], 0);
          }
          if ((rc = h2d(sa, m, hsrc(src_q), 0, m, h + a, cw)) < 0) return rc;
          cudaStreamWaitEvent(sc, mark_ev(sh), 0);
          cudaEvent_t seg = seg_begin(sc);
          rc = op_inner(c, prec, D, m, sa, m, m, w1, cw, sr, w1, so, w1, 0, sc);
          if (rc < 0) return rc;
          if ((rc = d2h_r(c0, h + a, w1, cw, sr, w1)) < 0) return rc;
          cudaEvent_t r_out = r_done;
          rc = op_outer(c, prec, D, m, so, w1, sa, m, m, w1, cw, sc);
          if (rc < 0) return rc;
          seg_end(2, sc, seg);
          wait(sd, sc);
          if ((rc = d2h(Q, 0, m, h + a, cw, sa, m)) < 0) return rc;
          cudaEvent_t out = mark_ev(sd);
          if (r_out) cudaStreamWaitEvent(sd, r_out, 0);   // (the slot's R12 is out too)
          freed[k] = r_out ? mark_ev(sd) : out;
        }
      }
      join_all();
      c->arena.release(mark);
    }
    return RGSQR_OK;
  }
};

}  // namespace

int factor_host(Ctx* c, const void* A, int64_t lda, int64_t m, int64_t n, void* Q, float* R, int prec,
                size_t budget) {
  int rc = validate(c, A, lda, m, n, Q, prec);
  if (rc < 0) return rc;
  if (!R && c->rank == 0) return fail(c, RGSQR_ERR_INVALID_ARG, "null R_out");
  if (c->opt.vshards > 1) return fail(c, RGSQR_ERR_UNSUPPORTED, "virtual shards: device path only");
  {
    // Device tiles use ld = m, and TMA needs 16-byte row pitches: a ragged m is staged through a
    // pinned bounce buffer of md = round_up(m, 16 / s) rows whose extra rows are zero.  Zero rows change
    // nothing: [A; 0] = [Q; 0] R (every dot product and norm is the same sum plus zeros).
    const int64_t s0 = elem_bytes(prec);
    if ((m * s0) % 16 != 0) {
      const int64_t md = (m * s0 + 15) / 16 * 16 / s0;
      void *Ab = nullptr, *Qb = nullptr;
      if (cudaHostAlloc(&Ab, (size_t)md * n * s0, cudaHostAllocPortable) != cudaSuccess ||
          cudaHostAlloc(&Qb, (size_t)md * n * s0, cudaHostAllocPortable) != cudaSuccess) {
        cudaGetLastError();
        if (Ab) cudaFreeHost(Ab);
        return fail(c, RGSQR_ERR_HOST_MEM, "ragged m: no pinned memory for the zero-padded bounce buffers");
      }
      for (int64_t j = 0; j < n; ++j) {
        char* d = static_cast<char*>(Ab) + (size_t)j * md * s0;
        std::memcpy(d, static_cast<const char*>(A) + (size_t)j * lda * s0, (size_t)m * s0);
        std::memset(d + (size_t)m * s0, 0, (size_t)(md - m) * s0);
      }
      const int64_t g0 = c->opt.graph;   // (per-call bounce buffers: no graph to reuse)
      c->opt.graph = 0;
      rc = factor_host(c, Ab, md, md, n, Qb, R, prec, budget);
      c->opt.graph = g0;
      if (rc >= 0)
        for (int64_t j = 0; j < n; ++j)
          std::memcpy(static_cast<char*>(Q) + (size_t)j * lda * s0, static_cast<char*>(Qb) + (size_t)j * md * s0,
                      (size_t)m * s0);
      cudaFreeHost(Ab);
      cudaFreeHost(Qb);
      return rc;
    }
  }
  reset_stats(c);
  rc = sync_shape(c, m, &budget);
  if (rc < 0) return rc;
  c->begin_call();
  const int s = elem_bytes(prec);

  // ---- page-lock caller buffers (timed separately) ----
  auto tp0 = std::chrono::steady_clock::now();
  std::vector<void*> registered;
  auto pin = [&](const void* p, size_t bytes) -> int {
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
      cudaGetLastError();
      at.type = cudaMemoryTypeUnregistered;
    }
    if (at.type == cudaMemoryTypeUnregistered) {
      for (void* q : registered)
        if (q == p) return RGSQR_OK;
      if (cudaHostRegister(const_cast<void*>(p), bytes, cudaHostRegisterPortable) != cudaSuccess) {
        cudaGetLastError();
        return fail(c, RGSQR_ERR_HOST_MEM, "cudaHostRegister failed");
      }
      registered.push_back(const_cast<void*>(p));
    }
    return RGSQR_OK;
  };
  const size_t abytes = ((size_t)lda * (n - 1) + m) * s;
  if ((rc = pin(A, abytes)) < 0 || (rc = pin(Q, abytes)) < 0 || (R && (rc = pin(R, (size_t)n * n * 4)) < 0)) {
    for (void* p : registered) cudaHostUnregister(p);
    return rc;
  }
  auto tp1 = std::chrono::steady_clock::now();

  // ---- device arena = the budget ----
  size_t cap = resolve_budget(c, budget);
  cap = cap > c->ctx_bytes ? cap - c->ctx_bytes : 0;   // context buffers count against the budget
  auto t0 = std::chrono::steady_clock::now();
  rc = ensure_arena(c, cap);
  if (rc < 0) {
    for (void* p : registered) cudaHostUnregister(p);
    return rc;
  }
  Exec x{c, prec, s, static_cast<const char*>(A), static_cast<char*>(Q), lda, m, n, R,
         c->compute(), c->st_h2d, c->st_d2h, c->st_d2r, (int)c->opt.ring_depth, c->opt.tile_rows_min,
         c->opt.tile_rows_max, c->opt.reuse != 0, c->opt.reorth != 0};
  x.sh2 = c->st_h2d2;
  if (c->opt.serialize) x.sh = x.sd = x.sr = x.sh2 = x.sc;
  // make the copy streams start after prior work of the compute stream
  x.join_all();
  cudaEvent_t t_ref = c->ev();
  cudaEventRecord(t_ref, x.sc);
  std::thread zero;
  if (R)
    zero = std::thread([R, n] {
      for (int64_t j = 0; j + 1 < n; ++j) std::memset(R + j * n + j + 1, 0, (size_t)(n - j - 1) * 4);
    });
  auto schedule = [&]() -> int {
    RGSQR_CUDA(c, cudaMemsetAsync(c->d_breakdown, 0x7f, sizeof(int), x.sc));
    return c->opt.algo == 1   ? x.blocked(std::min<int64_t>(c->opt.block_cols, n))
           : c->opt.algo == 2 ? x.fused_blocked(std::min<int64_t>(c->opt.block_cols, n))
                              : x.node(0, n, false);
  };
  // CUDA-graph replay (graph.cu) when the caller's buffers were already page-locked (the captured
  // copies address them directly; buffers this call registered are unregistered at its end)
  if (graph_allowed(c) && registered.empty()) {
    auto key = graph_key(c, 2, {reinterpret_cast<int64_t>(A), reinterpret_cast<int64_t>(Q),
                                reinterpret_cast<int64_t>(R), lda, m, n, prec});
    GraphEntry* g = graph_find(c, key);
    if (!g && !graph_known_bad(c, key)) {
      unsigned cnt0[2];
      const size_t amark = c->arena.mark();
      if (graph_capture_begin(c, x.sc, cnt0)) {
        x.fork_from_compute();
        int src = schedule();
        if (src >= 0) x.join_into_compute();
        graph_capture_end(c, x.sc, std::move(key), cnt0, src, &g);
        if (!g) {   // capture failed: nothing ran, re-run eagerly
          c->arena.release(amark);
          reset_stats(c);
        }
      }
    }
    rc = g ? graph_launch(c, g, x.sc) : schedule();
  } else {
    rc = schedule();
  }
  int brk = INT_MAX;
  if (rc >= 0) {
    x.join_all();
    cudaMemcpyAsync(&brk, c->d_breakdown, sizeof(int), cudaMemcpyDeviceToHost, x.sc);
  }
  cudaError_t e1 = cudaStreamSynchronize(x.sc);
  cudaError_t e2 = cudaStreamSynchronize(c->st_h2d);
  cudaError_t e3 = cudaStreamSynchronize(c->st_d2h);
  if (e3 == cudaSuccess) e3 = cudaStreamSynchronize(c->st_d2r);
  if (zero.joinable()) zero.join();
  auto t1 = std::chrono::steady_clock::now();
  for (void* p : registered) cudaHostUnregister(p);
  if (rc < 0) return rc;
  if (e1 != cudaSuccess || e2 != cudaSuccess || e3 != cudaSuccess)
    return fail(c, RGSQR_ERR_CUDA, std::string("stream error: ") +
                                       cudaGetErrorString(e1 != cudaSuccess ? e1 : (e2 != cudaSuccess ? e2 : e3)));
  // ---- stats ----
  auto& st = c->stats;
  st.pin_ms = std::chrono::duration<double, std::milli>(tp1 - tp0).count();
  st.wall_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
  // optional per-stream timeline (the paper's Figs. 8/10/13 as CSV): RGSQR_TIMELINE=path
  if (const char* tl = getenv("RGSQR_TIMELINE")) {
    if (FILE* f = fopen(tl, "w")) {
      fprintf(f, "stream,start_ms,end_ms\n");
      const char* nm[3] = {"h2d", "d2h", "compute"};
      for (auto& sg : c->segs) {
        float a = 0, b = 0;
        cudaEventElapsedTime(&a, t_ref, sg.a);
        cudaEventElapsedTime(&b, t_ref, sg.b);
        fprintf(f, "%s,%.4f,%.4f\n", nm[sg.kind], a, b);
      }
      fclose(f);
    }
  }
  for (auto& sg : c->segs) {
    float ms = 0;
    cudaEventElapsedTime(&ms, sg.a, sg.b);
    (sg.kind == 0 ? st.h2d_busy_ms : sg.kind == 1 ? st.d2h_busy_ms : st.compute_busy_ms) += ms;
  }
  const double sum = st.h2d_busy_ms + st.d2h_busy_ms + st.compute_busy_ms;
  const double mx = std::max({st.h2d_busy_ms, st.d2h_busy_ms, st.compute_busy_ms});
  st.overlap_ratio = sum - mx > 1e-9 ? std::min(1.0, std::max(0.0, (sum - st.wall_ms) / (sum - mx))) : 0.0;
  st.arena_bytes = (int64_t)c->arena.size;
  st.arena_high_water = (int64_t)c->arena.high;
  st.ctx_device_bytes = (int64_t)c->ctx_bytes;
  st.flops = (int64_t)(2.0 * m * (double)n * n);
  if (brk == -2) {
    c->broken = true;
    return fail(c, RGSQR_ERR_CUDA, "leaf exchange timed out (a rank did not arrive)");
  }
  st.first_breakdown_col = (brk == 0x7f7f7f7f || brk == INT_MAX) ? -1 : brk;
  c->collect_kernel_stats();
  return st.first_breakdown_col >= 0 ? RGSQR_WARN_RANK_DEFICIENT : RGSQR_OK;
}

}  // namespace rgsqr
