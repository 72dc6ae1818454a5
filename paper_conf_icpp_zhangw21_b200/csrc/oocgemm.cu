// oocgemm.cu -- the two out-of-core GEMMs of the method as standalone operations, with both tiling
// strategies the paper compares (section 3.3; measured in Tables 1/2,
// PAPER.md:255-301):
//
//   inner product  R12 = Q1^T A2   (TN; Q1 m x w1, A2 m x w2 in host memory, R12 w1 x w2 fp32)
//     tiling 0 (recursive, Fig. 3): row tiles of t rows of BOTH operands stream through the device,
//              each read once; R12 accumulates in HBM and goes out once at the end.
//     tiling 1 (blocking, Fig. 4):  Q1 (the panel) resident, A2 in column blocks of b columns; each
//              block's R12 block goes out as soon as it is done.
//   outer product  A2 <- A2 - Q1 R12   (NN; A2 updated in place in host memory)
//     tiling 0 (recursive, Fig. 5): R12 resident, row tiles of Q1 and A2 in, A2' tiles out.
//     tiling 1 (blocking, Fig. 6):  Q1 and R12 resident, b x b tiles of A2 in and out.
//
// Every tile moves through a K-slot device ring on the library's three streams (H2D, compute, D2H),
// chained by events: loaded[s] -> kernel -> computed[s] -> D2H -> free[s] -> next upload into s.
// RGSQR_OPT_SERIALIZE runs everything on one stream: the paper's "Synchronous" rows.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <algorithm>
#include <chrono>
#include <vector>

#include "engine.h"

namespace rgsqr {
int ensure_arena(Ctx* c, size_t want);
size_t resolve_budget(Ctx* c, size_t budget);
void reset_stats(Ctx* c);

namespace {

struct Pipe {
  Ctx* c;
  cudaStream_t sc, sh, sd;
  int64_t s;
  std::vector<cudaEvent_t> freed;   // per slot: the slot may be overwritten after this event
  // (inside a graph capture: timed only for RGSQR_TIMELINE, as external event record nodes)
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
    if (c->capturing && !c->graph_timeline) return nullptr;
    return seg_event(st);
  }
  void seg_end(int kind, cudaStream_t st, cudaEvent_t a) {
    if (!a) return;
    c->segs.push_back({kind, a, seg_event(st)});
  }
  cudaEvent_t mark(cudaStream_t st) {
    cudaEvent_t e = c->ev();
    cudaEventRecord(e, st);
    return e;
  }
  // rows x cols block of a column-major host matrix (ld) <-> device (ldd)
  int up(void* dst, int64_t ldd, const char* src, int64_t ld, int64_t r0, int64_t c0, int64_t rows, int64_t cols,
         int64_t esz) {
    cudaEvent_t a = seg_begin(sh);
    RGSQR_CUDA(c, cudaMemcpy2DAsync(dst, ldd * esz, src + (r0 + c0 * ld) * esz, ld * esz, rows * esz, cols,
                                    cudaMemcpyHostToDevice, sh));
    seg_end(0, sh, a);
    c->stats.h2d_bytes += rows * cols * esz;
    c->stats.h2d_matrix_bytes += rows * cols * esz;
    return RGSQR_OK;
  }
  int down(char* dst, int64_t ld, int64_t r0, int64_t c0, const void* src, int64_t lds, int64_t rows, int64_t cols,
           int64_t esz) {
    cudaEvent_t a = seg_begin(sd);
    RGSQR_CUDA(c, cudaMemcpy2DAsync(dst + (r0 + c0 * ld) * esz, ld * esz, src, lds * esz, rows * esz, cols,
                                    cudaMemcpyDeviceToHost, sd));
    seg_end(1, sd, a);
    c->stats.d2h_bytes += rows * cols * esz;
    c->stats.d2h_matrix_bytes += rows * cols * esz;
    return RGSQR_OK;
  }
};

int cast_r12(Ctx* c, int prec, const float* src, int64_t lds, void* dst, int64_t ldd, int64_t M, int64_t N,
             cudaStream_t st) {
  cudaError_t e;
  switch (prec) {
    case RGSQR_FP16: e = launch_copy_cast<__half>(src, lds, nullptr, 0, static_cast<__half*>(dst), ldd, M, N, st); break;
    case RGSQR_BF16:
      e = launch_copy_cast<__nv_bfloat16>(src, lds, nullptr, 0, static_cast<__nv_bfloat16*>(dst), ldd, M, N, st);
      break;
    default: e = launch_copy_cast<float>(src, lds, nullptr, 0, static_cast<float*>(dst), ldd, M, N, st);
  }
  if (e != cudaSuccess) return fail(c, RGSQR_ERR_CUDA, std::string("R12 operand copy: ") + cudaGetErrorString(e));
  c->stats.n_other_launches++;
  return RGSQR_OK;
}

}  // namespace

// op: 0 inner, 1 outer.  Host arrays: Q1 (m x w1, ldq), A2 (m x w2, lda), R12 (w1 x w2 fp32, ldr).
int ooc_gemm(Ctx* c, int op, int tiling, int64_t block, const void* Q1, int64_t ldq, void* A2, int64_t lda,
             float* R12, int64_t ldr, int64_t m, int64_t w1, int64_t w2, int prec, size_t budget) {
  if (!Q1 || !A2 || !R12 || m < 1 || w1 < 1 || w2 < 1 || ldq < m || lda < m || ldr < w1 || (op != 0 && op != 1) ||
      (tiling != 0 && tiling != 1) || prec < RGSQR_FP16 || prec > RGSQR_TF32X3)
    return fail(c, RGSQR_ERR_INVALID_ARG, "ooc gemm: bad arguments");
  if (c->nccl_comm) return fail(c, RGSQR_ERR_UNSUPPORTED, "ooc gemm: single-GPU contexts only");
  if (prec == RGSQR_TF32X3) return fail(c, RGSQR_ERR_UNSUPPORTED, "ooc gemm: fp16 / bf16 / tf32 only");
  const int64_t s = elem_bytes(prec);
  if ((ldq * s) % 16 || (lda * s) % 16) return fail(c, RGSQR_ERR_INVALID_ARG, "ooc gemm: ld*sizeof(elem) % 16 != 0");
  reset_stats(c);
  c->begin_call();
  // page-lock pageable caller buffers for the call (cost in stats.pin_ms, excluded from wall_ms)
  std::vector<void*> registered;
  auto tp0 = std::chrono::steady_clock::now();
  auto pin = [&](const void* p, size_t bytes) -> bool {
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
      cudaGetLastError();
      at.type = cudaMemoryTypeUnregistered;
    }
    if (at.type != cudaMemoryTypeUnregistered) return true;
    if (cudaHostRegister(const_cast<void*>(p), bytes, cudaHostRegisterPortable) != cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    registered.push_back(const_cast<void*>(p));
    return true;
  };
  struct Unpin {   // (after every stream of the call has drained, also on error paths)
    Ctx* c;
    std::vector<void*>* v;
    ~Unpin() {
      cudaStreamSynchronize(c->compute());
      cudaStreamSynchronize(c->st_h2d);
      cudaStreamSynchronize(c->st_d2h);
      for (void* p : *v) cudaHostUnregister(p);
    }
  } unpin{c, &registered};
  if (!pin(Q1, ((size_t)ldq * (w1 - 1) + m) * s) || !pin(A2, ((size_t)lda * (w2 - 1) + m) * s) ||
      !pin(R12, ((size_t)ldr * (w2 - 1) + w1) * 4))
    return fail(c, RGSQR_ERR_HOST_MEM, "ooc gemm: cudaHostRegister failed");
  c->stats.pin_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tp0).count();
  size_t cap = resolve_budget(c, budget);
  cap = cap > c->ctx_bytes ? cap - c->ctx_bytes : 0;   // context buffers count against the budget
  int rc = ensure_arena(c, cap);
  if (rc < 0) return rc;
  Pipe P{c, c->compute(), c->st_h2d, c->st_d2h, s, {}};
  // device leading dimension of resident panels / column blocks: TMA needs 16-byte pitches, so a ragged m is
  // padded (the tensor maps keep m rows; the pad rows are never read)
  const int64_t md = (m * s + 15) / 16 * 16 / s;
  if (c->opt.serialize) P.sh = P.sd = P.sc;
  int K = (int)c->opt.ring_depth;   // (lowered to >= 2 slots when the budget is tight)
  P.freed.assign(K, nullptr);
  const char* hq = static_cast<const char*>(Q1);
  char* ha = static_cast<char*>(A2);
  char* hr = reinterpret_cast<char*>(R12);
  auto t0 = std::chrono::steady_clock::now();
  // start after prior work of the compute stream
  cudaEvent_t start = P.mark(P.sc);
  cudaStreamWaitEvent(P.sh, start, 0);
  cudaStreamWaitEvent(P.sd, start, 0);
  cudaEvent_t t_ref = start;
  const size_t ws_reserve = (size_t)16 << 20;   // split-K partials of the per-tile products
  auto fits_rows = [&](size_t resident, size_t per_row, int64_t want) -> int64_t {
    const size_t free_b = c->arena.free_bytes();
    if (free_b < resident + ws_reserve) return 0;
    for (; K >= 2; --K) {
      int64_t t = (int64_t)((free_b - resident - ws_reserve) / ((size_t)K * per_row));
      t = std::min<int64_t>({t, want, (m + 127) / 128 * 128}) / 128 * 128;
      if (t >= std::min<int64_t>(want, 1024) || K == 2) return t;
    }
    return 0;
  };
  auto fits_slots = [&](size_t per) -> bool {   // K column blocks / tiles of `per` bytes
    const size_t free_b = c->arena.free_bytes();
    while (K > 2 && (size_t)K * per + ws_reserve > free_b) --K;
    return (size_t)K * per + ws_reserve <= free_b;
  };
  auto schedule = [&]() -> int {
    if (op == 0 && tiling == 0) {
      // ---- Fig. 3: R12 resident (fp32), row tiles of Q1 and A2 ----
      float* dR = static_cast<float*>(c->arena.alloc((size_t)w1 * w2 * 4));
      const int64_t t = dR ? fits_rows(0, (size_t)(w1 + w2) * s, block > 0 ? block : 16384) : 0;
      if (!dR || t < 128) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "ooc inner: R12 + 2 tiles do not fit");
      char* ring = static_cast<char*>(c->arena.alloc((size_t)K * t * (w1 + w2) * s));
      if (!ring) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "ooc inner: ring");
      int64_t i = 0;
      for (int64_t r0 = 0; r0 < m; r0 += t, ++i) {
        const int64_t tr = std::min(t, m - r0);
        const int k = (int)(i % K);
        char* sq = ring + (size_t)k * t * (w1 + w2) * s;
        char* sa = sq + (size_t)t * w1 * s;
        if (P.freed[k]) cudaStreamWaitEvent(P.sh, P.freed[k], 0);
        if ((rc = P.up(sq, t, hq, ldq, r0, 0, tr, w1, s)) < 0) return rc;
        if ((rc = P.up(sa, t, ha, lda, r0, 0, tr, w2, s)) < 0) return rc;
        cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
        cudaEvent_t a = P.seg_begin(P.sc);
        rc = op_inner(c, prec, sq, t, sa, t, tr, w1, w2, dR, w1, nullptr, w1, i > 0 ? 1 : 0, P.sc, false);
        if (rc < 0) return rc;
        P.seg_end(2, P.sc, a);
        P.freed[k] = P.mark(P.sc);
      }
      cudaStreamWaitEvent(P.sd, P.mark(P.sc), 0);
      if ((rc = P.down(hr, ldr, 0, 0, dR, w1, w1, w2, 4)) < 0) return rc;
    } else if (op == 0) {
      // ---- Fig. 4: Q1 (the panel) resident, column blocks of A2, R12 blocks out ----
      const int64_t b = std::min<int64_t>(w2, block > 0 ? block : 16384);
      char* dQ = static_cast<char*>(c->arena.alloc((size_t)md * w1 * s));
      const size_t per = (size_t)md * b * s + (size_t)w1 * b * 4 + 512;
      if (!dQ || !fits_slots(per))
        return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "ooc inner (blocking): panel + 2 column blocks do not fit");
      char* ring = static_cast<char*>(c->arena.alloc((size_t)K * per));
      if ((rc = P.up(dQ, md, hq, ldq, 0, 0, m, w1, s)) < 0) return rc;
      cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
      int64_t i = 0;
      for (int64_t c0 = 0; c0 < w2; c0 += b, ++i) {
        const int64_t bw = std::min(b, w2 - c0);
        const int k = (int)(i % K);
        char* sa = ring + (size_t)k * per;
        float* sr = reinterpret_cast<float*>(sa + (size_t)md * b * s);
        if (P.freed[k]) cudaStreamWaitEvent(P.sh, P.freed[k], 0);
        if ((rc = P.up(sa, md, ha, lda, 0, c0, m, bw, s)) < 0) return rc;
        cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
        if (P.freed[k]) cudaStreamWaitEvent(P.sc, P.freed[k], 0);   // the block's previous R12 is out
        cudaEvent_t a = P.seg_begin(P.sc);
        rc = op_inner(c, prec, dQ, md, sa, md, m, w1, bw, sr, w1, nullptr, w1, 0, P.sc, false);
        if (rc < 0) return rc;
        P.seg_end(2, P.sc, a);
        cudaStreamWaitEvent(P.sd, P.mark(P.sc), 0);
        if ((rc = P.down(hr, ldr, 0, c0, sr, w1, w1, bw, 4)) < 0) return rc;
        P.freed[k] = P.mark(P.sd);
      }
    } else {
      // ---- outer product: R12 uploaded once (fp32) and rounded to the operand type on the device ----
      char* dRop = static_cast<char*>(c->arena.alloc((size_t)w1 * w2 * s));
      const size_t mk = c->arena.mark();
      float* dRf = static_cast<float*>(c->arena.alloc((size_t)w1 * std::min<int64_t>(w2, 4096) * 4));
      if (!dRop || !dRf) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "ooc outer: R12 does not fit");
      for (int64_t c0 = 0; c0 < w2; c0 += 4096) {   // (staged in 4096-column pieces)
        const int64_t cw = std::min<int64_t>(4096, w2 - c0);
        if ((rc = P.up(dRf, w1, hr, ldr, 0, c0, w1, cw, 4)) < 0) return rc;
        cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
        if ((rc = cast_r12(c, prec, dRf, w1, dRop + (size_t)c0 * w1 * s, w1, w1, cw, P.sc)) < 0) return rc;
        cudaStreamWaitEvent(P.sh, P.mark(P.sc), 0);
      }
      c->arena.release(mk);
      if (tiling == 0) {
        // ---- Fig. 5: row tiles of Q1 and A2 in, A2' tiles out ----
        const int64_t t = fits_rows(0, (size_t)(w1 + w2) * s, block > 0 ? block : 8192);
        if (t < 128) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "ooc outer: R12 + 2 tiles do not fit");
        char* ring = static_cast<char*>(c->arena.alloc((size_t)K * t * (w1 + w2) * s));
        int64_t i = 0;
        for (int64_t r0 = 0; r0 < m; r0 += t, ++i) {
          const int64_t tr = std::min(t, m - r0);
          const int k = (int)(i % K);
          char* sq = ring + (size_t)k * t * (w1 + w2) * s;
          char* sa = sq + (size_t)t * w1 * s;
          if (P.freed[k]) cudaStreamWaitEvent(P.sh, P.freed[k], 0);
          if ((rc = P.up(sq, t, hq, ldq, r0, 0, tr, w1, s)) < 0) return rc;
          if ((rc = P.up(sa, t, ha, lda, r0, 0, tr, w2, s)) < 0) return rc;
          cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
          cudaEvent_t a = P.seg_begin(P.sc);
          rc = op_outer(c, prec, sq, t, dRop, w1, sa, t, tr, w1, w2, P.sc);
          if (rc < 0) return rc;
          P.seg_end(2, P.sc, a);
          cudaStreamWaitEvent(P.sd, P.mark(P.sc), 0);
          if ((rc = P.down(ha, lda, r0, 0, sa, t, tr, w2, s)) < 0) return rc;
          P.freed[k] = P.mark(P.sd);
        }
      } else {
        // ---- Fig. 6: Q1 resident too, b x b tiles of A2 in and out ----
        const int64_t b = block > 0 ? block : 16384;
        const int64_t b1 = std::min(b, (m + 127) / 128 * 128), b2 = std::min(b, w2);
        char* dQ = static_cast<char*>(c->arena.alloc((size_t)md * w1 * s));
        const size_t per = (size_t)b1 * b2 * s;
        if (!dQ || !fits_slots(per))
          return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "ooc outer (blocking): Q1 + R12 + 2 tiles do not fit");
        char* ring = static_cast<char*>(c->arena.alloc((size_t)K * per));
        if ((rc = P.up(dQ, md, hq, ldq, 0, 0, m, w1, s)) < 0) return rc;
        cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
        int64_t i = 0;
        for (int64_t r0 = 0; r0 < m; r0 += b1)
          for (int64_t c0 = 0; c0 < w2; c0 += b2, ++i) {
            const int64_t tr = std::min(b1, m - r0), tc = std::min(b2, w2 - c0);
            const int k = (int)(i % K);
            char* sa = ring + (size_t)k * per;
            if (P.freed[k]) cudaStreamWaitEvent(P.sh, P.freed[k], 0);
            if ((rc = P.up(sa, b1, ha, lda, r0, c0, tr, tc, s)) < 0) return rc;
            cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
            cudaEvent_t a = P.seg_begin(P.sc);
            rc = op_outer(c, prec, dQ + (size_t)r0 * s, md, dRop + (size_t)c0 * w1 * s, w1, sa, b1, tr, w1, tc, P.sc);
            if (rc < 0) return rc;
            P.seg_end(2, P.sc, a);
            cudaStreamWaitEvent(P.sd, P.mark(P.sc), 0);
            if ((rc = P.down(ha, lda, r0, c0, sa, b1, tr, tc, s)) < 0) return rc;
            P.freed[k] = P.mark(P.sd);
          }
      }
    }
    return RGSQR_OK;
  };
  // CUDA-graph replay (graph.cu, R30) when the caller's buffers were already page-locked
  if (graph_allowed(c) && registered.empty()) {
    auto key = graph_key(c, 3, {op, tiling, block, reinterpret_cast<int64_t>(Q1), reinterpret_cast<int64_t>(A2),
                                reinterpret_cast<int64_t>(R12), ldq, lda, ldr, m, w1, w2, prec});
    GraphEntry* g = graph_find(c, key);
    if (!g && !graph_known_bad(c, key)) {
      unsigned cnt0[2];
      const size_t amark = c->arena.mark();
      const int K0 = K;
      if (graph_capture_begin(c, P.sc, cnt0)) {
        cudaEvent_t f = P.mark(P.sc);   // the copy streams join the capture
        cudaStreamWaitEvent(P.sh, f, 0);
        cudaStreamWaitEvent(P.sd, f, 0);
        int src = schedule();
        if (src >= 0) {
          cudaStreamWaitEvent(P.sc, P.mark(P.sh), 0);
          cudaStreamWaitEvent(P.sc, P.mark(P.sd), 0);
        }
        graph_capture_end(c, P.sc, std::move(key), cnt0, src, &g);
        if (!g) {   // capture failed: nothing ran, re-run eagerly
          const double pin_ms = c->stats.pin_ms;
          c->arena.release(amark);
          reset_stats(c);
          c->stats.pin_ms = pin_ms;
          K = K0;
          P.freed.assign(K, nullptr);
        }
      }
    }
    rc = g ? graph_launch(c, g, P.sc) : schedule();
  } else {
    rc = schedule();
  }
  if (rc < 0) return rc;
  cudaError_t e1 = cudaStreamSynchronize(P.sc);
  cudaError_t e2 = cudaStreamSynchronize(c->st_h2d);
  cudaError_t e3 = cudaStreamSynchronize(c->st_d2h);
  auto t1 = std::chrono::steady_clock::now();
  if (e1 != cudaSuccess || e2 != cudaSuccess || e3 != cudaSuccess)
    return fail(c, RGSQR_ERR_CUDA, std::string("ooc gemm: ") +
                                       cudaGetErrorString(e1 != cudaSuccess ? e1 : (e2 != cudaSuccess ? e2 : e3)));
  auto& st = c->stats;
  st.wall_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
  (void)st.pin_ms;
  for (auto& sg : c->segs) {
    float ms = 0;
    cudaEventElapsedTime(&ms, sg.a, sg.b);
    (sg.kind == 0 ? st.h2d_busy_ms : sg.kind == 1 ? st.d2h_busy_ms : st.compute_busy_ms) += ms;
  }
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
  const double sum = st.h2d_busy_ms + st.d2h_busy_ms + st.compute_busy_ms;
  const double mx = std::max({st.h2d_busy_ms, st.d2h_busy_ms, st.compute_busy_ms});
  st.overlap_ratio = sum - mx > 1e-9 ? std::min(1.0, std::max(0.0, (sum - st.wall_ms) / (sum - mx))) : 0.0;
  st.arena_bytes = (int64_t)c->arena.size;
  st.arena_high_water = (int64_t)c->arena.high;
  st.ctx_device_bytes = (int64_t)c->ctx_bytes;
  st.flops = (int64_t)(2.0 * (double)m * w1 * w2);
  c->collect_kernel_stats();
  return RGSQR_OK;
}

}  // namespace rgsqr
