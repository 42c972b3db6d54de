// runtime.cpp -- device side of the engine and the extern "C" entry points of include/bm.h.
//
// Launch path (A5, §5 "Keeping the GPU busy", L391): every task of one Schedule call is
// staged in a pinned host ring of 16-byte row descriptors, copied to the device with ONE
// cudaMemcpyAsync, and all kernels of all tasks are pushed onto one stream in order, without
// waiting. After each task a signal kernel bumps a counter in mapped pinned host memory
// (§5 "Asynchronous Completion Notification", L393-L395); bm_poll / the run loop compare the
// counter against the in-progress FIFO and retire finished tasks in order.
#include <cuda_bf16.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <functional>
#include <new>
#include <thread>

#include "engine.h"

namespace bm {

long long realtime_ns() {
  timespec ts;
  clock_gettime(CLOCK_REALTIME, &ts);
  return static_cast<long long>(ts.tv_sec) * 1000000000LL + ts.tv_nsec;
}

double wall_now(const Engine& e) {
  return std::chrono::duration<double>(std::chrono::steady_clock::now() - e.t0).count();
}

namespace {

// A failing CUDA call makes the engine unusable (BM_E_CUDA is sticky, include/bm.h); the
// failing call and the CUDA error are reported on stderr once.
#define CK(x)                                                                                  \
  do {                                                                                         \
    cudaError_t err__ = (x);                                                                   \
    if (err__ != cudaSuccess) {                                                                \
      if (!e.sticky_cuda)                                                                      \
        fprintf(stderr, "bm: %s:%d: %s -> %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(err__)); \
      e.sticky_cuda = true;                                                                    \
      return BM_E_CUDA;                                                                        \
    }                                                                                          \
  } while (0)

template <class T>
cudaError_t dalloc(T** p, size_t n) {
  return cudaMalloc(reinterpret_cast<void**>(p), n * sizeof(T));
}

// Algorithmic bytes / flops of one cell-step launch: weights streamed
// once, gathered operand rows, state read/written, result rows. Padding is not counted.
void algo_cost(const Engine& e, const Cell& c, int b, bool proj, double* bytes, double* flops) {
  const double H = static_cast<double>(e.cfg.hidden);
  const double el = static_cast<double>(e.elem());
  if (proj) {
    const double V = c.d.vocab;
    *bytes = V * H * el + V * 4 + b * (H * el + 8.0);
    *flops = 2.0 * b * H * V;
    return;
  }
  const double K = c.K0 + c.K1;
  const double rows = static_cast<double>(c.G) * H;
  double per_row = K * el + H * el + H * 4;              // gather, h' write, c' write
  if (c.epi == EPI_LSTM) per_row += H * 4;                // c read
  if (c.epi == EPI_INTERNAL) per_row += 2 * H * 4;        // c_L, c_R read
  *bytes = rows * K * el + rows * 4 + b * per_row;
  *flops = 2.0 * b * K * rows;
}

// Host half of the per-kernel roofline (include/bm.h "measurement"): the launch's algorithmic
// bytes / flops and its time at each roof, added to its kernel class.
void account_launch(Engine& e, int kc, int b, double bytes, double flops) {
  bm_stats& s = e.stats;
  s.k_launches[kc] += 1;
  s.k_rows[kc] += b;
  s.k_bytes[kc] += bytes;
  s.k_flops[kc] += flops;
  const double t_hbm = e.cfg.roof_hbm_gbs > 0 ? bytes / (e.cfg.roof_hbm_gbs * 1e6) : 0.0;   // ms
  const double t_tc = e.cfg.roof_tc_tflops > 0 ? flops / (e.cfg.roof_tc_tflops * 1e9) : 0.0;  // ms
  s.k_roof_hbm_ms[kc] += t_hbm;
  s.k_roof_tc_ms[kc] += t_tc;
  s.k_roof_ms[kc] += std::max(t_hbm, t_tc);
}

}  // namespace

// ---------------------------------------------------------------- workers (§8f N2)
static void swap_active(Engine& e, WorkerState& w) {
  std::swap(e.stream, w.stream);
  std::swap(e.inflight, w.inflight);
  std::swap(e.launched, w.launched);
  std::swap(e.last_finish, w.last_finish);
  std::swap(e.signal_host, w.signal_host);
  std::swap(e.signal_dev, w.signal_dev);
  std::swap(e.dep_flag, w.dep_flag);
  std::swap(e.dep_seq, w.dep_seq);
  std::swap(e.pdl_ok, w.pdl_ok);
  std::swap(e.sig_ctas, w.sig_ctas);
  std::swap(e.done_ctas, w.done_ctas);
  std::swap(e.amax, w.amax);
  std::swap(e.scratch, w.scratch);
}

// Device contexts (§8f N2): swap the active context's pool / ring / weights with a parked one.
static void swap_ctx(Engine& e, DevCtx& c) {
  std::swap(e.h_pool, c.h_pool);
  std::swap(e.c_pool, c.c_pool);
  std::swap(e.tok, c.tok);
  std::swap(e.dead, c.dead);
  std::swap(e.ring_dev, c.ring_dev);
  std::swap(e.ring_host, c.ring_host);
  std::swap(e.ring_head, c.ring_head);
  std::swap(e.rows_flag_dev, c.rows_flag_dev);
  std::swap(e.rows_seq_host, c.rows_seq_host);
  std::swap(e.rows_seq, c.rows_seq);
  std::swap(e.copy_stream, c.copy_stream);
  std::swap(e.copy_ev, c.copy_ev);
  c.cells.resize(e.cells.size());
  for (size_t i = 0; i < e.cells.size(); ++i) {
    Cell& a = e.cells[i];
    CellWeights& b = c.cells[i];
    std::swap(a.W, b.W);
    std::swap(a.bias, b.bias);
    std::swap(a.E, b.E);
    std::swap(a.W_out, b.W_out);
    std::swap(a.b_out, b.b_out);
  }
}

static void select_ctx(Engine& e, int c) {
  if (c == e.cur_ctx || e.ctxs.size() < 2) return;
  swap_ctx(e, e.ctxs[e.cur_ctx]);
  swap_ctx(e, e.ctxs[c]);
  e.cur_ctx = c;
  if (e.device()) cudaSetDevice(e.ctxs[c].cuda_dev);
}

// Make worker w's launch state (and its device context) the engine's active one (no-op with
// one worker).
void select_worker(Engine& e, int w) {
  if (w == e.cur || e.parked.empty()) return;
  swap_active(e, e.parked[e.cur]);
  swap_active(e, e.parked[w]);
  e.cur = w;
  select_ctx(e, e.worker_ctx.empty() ? 0 : e.worker_ctx[w]);
}

// §8f N2 state migration (L337): before a task runs on the active context, every input state
// row it reads that another context wrote last (its subgraph moved: unpinned, nothing in
// flight, L381) is copied over -- h of both parities and c of every pool layer, the feed token
// and the <eos> mark -- on the active worker's stream, ahead of the task's kernels. The producer
// of that state has retired (pinning), so its writes are complete.
static bm_status migrate_inputs(Engine& e, std::vector<Task>& tasks) {
  if (e.ctxs.size() < 2) return BM_OK;
  const int to = e.cur_ctx;
  const size_t H = e.H(), S = e.cfg.max_slots, L = e.cfg.pool_layers, el = e.elem();
  auto move = [&](int slot) -> bm_status {
    const int from = e.slot_ctx[slot];
    if (from < 0 || from == to) return BM_OK;
    e.stats.migrations += 1;
    e.stats.migration_bytes += static_cast<double>(L * (2 * H * el + H * 4) + 8);
    if (e.device()) {
      const DevCtx& src = e.ctxs[from];
      const int dd = e.ctxs[to].cuda_dev, sd = src.cuda_dev;
      for (size_t l = 0; l < L; ++l) {
        for (size_t par = 0; par < 2; ++par) {
          const size_t off = ((l * 2 + par) * S + slot) * H * el;
          CK(cudaMemcpyPeerAsync(static_cast<char*>(e.h_pool) + off, dd, static_cast<const char*>(src.h_pool) + off,
                                 sd, H * el, e.stream));
        }
        const size_t coff = (l * S + slot) * H;
        CK(cudaMemcpyPeerAsync(e.c_pool + coff, dd, src.c_pool + coff, sd, H * 4, e.stream));
      }
      CK(cudaMemcpyPeerAsync(e.tok + slot, dd, src.tok + slot, sd, 4, e.stream));
      CK(cudaMemcpyPeerAsync(e.dead + slot, dd, src.dead + slot, sd, 4, e.stream));
      e.pdl_ok = false;  // copies precede the next launch on this stream: full ordering
    }
    return BM_OK;
  };
  for (Task& t : tasks) {
    const int epi = e.cells[t.ct].epi;
    for (const RowDesc& r : t.desc) {
      bm_status st = BM_OK;
      if (epi == EPI_INTERNAL) {          // children's h / c by slot
        st = move(r.a);
        if (st == BM_OK) st = move(r.b);
      } else if (epi == EPI_LSTM && !(r.flags & ROW_FIRST)) {  // the request's own state
        st = move(r.slot);
      }
      if (st != BM_OK) return st;
    }
    for (const RowDesc& r : t.desc) e.slot_ctx[r.slot] = static_cast<int8_t>(to);
  }
  return BM_OK;
}

// ---------------------------------------------------------------- launching tasks
static bm_status launch_one_step(Engine& e, Cell& c, const RowDesc* rows_dev, const RowDesc* rows_host,
                                 int b, int layer, bool proj, unsigned long long* signal,
                                 unsigned long long sig_value = 0) {
  StepArgs a{};
  a.epi = proj ? EPI_PROJ : c.epi;
  a.G = proj ? 1 : c.G;
  a.H = e.cfg.hidden;
  a.K0 = c.K0;
  a.K1 = proj ? 0 : c.K1;
  a.U = c.U;
  // split-K factor per launch (bf16 path): 512-wide K slices up to 256 rows (one wave of
  // 128-160 CTAs); above that two column blocks with 1024-wide slices keep one wave instead of
  // two (the wider K slice costs less than a second wave and halves the DSMEM exchange).
  a.S = c.S;
  if (e.cfg.precision == BM_PREC_BF16 && b > 256 && c.S >= 4) a.S = c.S / 2;
  a.kslice = (c.K0 + c.K1) / a.S;
  if (proj) {
    a.S = 1;
    a.kslice = e.cfg.hidden;
  }
  a.b = b;
  a.layer = layer;
  a.n_slots = e.cfg.max_slots;
  a.rows = rows_dev;
  a.E = c.E;
  a.V = c.d.vocab;
  const bool tree = c.epi == EPI_LEAF || c.epi == EPI_INTERNAL;
  const int pl = tree ? 0 : (proj ? c.d.layers - 1 : layer);
  a.h_lower = (!tree && !proj && layer > 0) ? e.h_layer(layer - 1) : nullptr;
  a.h_pool = e.h_layer(pl);
  a.c_pool = e.c_layer(pl);
  a.tok = e.tok;
  a.dead = e.dead;
  a.eos_host = e.eos_dev;
  a.small_plan = e.cfg.workers > 1 ? 1 : 0;  // two workers' CTAs share the SMs
  a.W = proj ? c.W_out : c.W[layer];
  a.bias = proj ? c.b_out : c.bias[layer];
  a.W_rows = proj ? c.d.vocab : c.G * e.cfg.hidden;
  a.res_h = e.res_h;
  a.res_c = e.res_c;
  a.res_layers = e.cfg.pool_layers;
  a.amax = e.amax;
  a.scratch = e.scratch;
  a.done_ctas = e.done_ctas;
  a.res_tok = e.res_tok;
  a.max_decode = e.cfg.max_decode_len;
  a.logits = (proj && e.logits != nullptr) ? e.logits : nullptr;
  a.phase = e.phase_dev;
  static const int max_stages = getenv("BM_MAX_STAGES") ? atoi(getenv("BM_MAX_STAGES")) : 0;
  a.max_stages = max_stages;
  static const int experiment = getenv("BM_EXPERIMENT") ? atoi(getenv("BM_EXPERIMENT")) : 0;
  a.experiment = experiment;
  a.signal = signal;
  a.sig_value = sig_value;
  a.sig_ctas = e.sig_ctas;
  // PDL only directly behind another tcgen05 launch: the chain flag orders launches among
  // themselves, while copies / other kernels before a launch need full stream ordering
  static const int no_pdl = getenv("BM_NO_PDL") ? atoi(getenv("BM_NO_PDL")) : 0;
  static const int no_chain = getenv("BM_NO_CHAIN") ? atoi(getenv("BM_NO_CHAIN")) : 0;
  a.pdl = (no_pdl || !e.pdl_ok) ? 0 : 1;
  if (!no_chain) {
    a.dep_flag = e.dep_flag;
    a.dep_seq = e.dep_seq + 1;
  }
  if (rows_dev != nullptr && e.launch_rows_seq != 0) {
    a.rows_flag = e.rows_flag_dev;
    a.rows_seq = e.launch_rows_seq;
  }
  // time_kernels: EVERY launch gets a device span slot, its class accumulator and a log entry
  const bool timed = e.cfg.time_kernels && e.spans != nullptr;
  uint64_t log_i = 0;
  if (timed) {
    const uint64_t i = e.timed_total++;
    log_i = i % Engine::kLaunchLog;
    a.span = e.spans + 2 * (i % 64);   // PDL keeps at most a few launches open at once
    a.span_acc = e.spans + 128;        // class accumulators: the launcher offsets by class
    a.span_log = e.span_log + log_i;
  }
  if (e.tl_dev != nullptr && e.tl_n < Engine::kTimeline) {
    a.tl = e.tl_dev + 4 * e.tl_n;
    e.tl_host[e.tl_n] = realtime_ns();
    e.tl_b[e.tl_n] = b;
    e.tl_n += 1;
  }
  cudaError_t err;
  int kc = BM_K_SIMT;
  if (e.cfg.precision == BM_PREC_BF16) {
    err = launch_cell_step_sm100(a, rows_host, e.stream, &kc);
    if (err == cudaSuccess) {
      if (!no_chain) e.dep_seq += 1;
      e.pdl_ok = true;
    }
  } else {
    a.pdl = 0;  // the SIMT kernels do not use griddepcontrol
    if (timed) a.span_acc += 2 * BM_K_SIMT;
    err = launch_cell_step_simt(a, e.stream);
  }
  CK(err);
  if (timed) {
    double bytes, flops;
    algo_cost(e, c, b, proj, &bytes, &flops);
    account_launch(e, kc, b, bytes, flops);
    e.launch_class[log_i] = kc;
    e.launch_b[log_i] = b;
  }
  e.stats.kernel_launches += 1;
  return BM_OK;
}

// All kernels of one task in order on the engine stream (§5). With `signal`, the task's
// completion is signalled: fused into the last kernel's last CTA on the tcgen05 path (A12),
// or by the signal kernel on the fp32 path.
static bm_status launch_cell(Engine& e, Cell& c, const RowDesc* rows_dev, const RowDesc* rows_host, int b,
                             Task* t, unsigned long long* signal) {
  const bool lstm = c.epi == EPI_LSTM;
  const bool proj = c.d.kind == BM_CELL_LSTM_PROJ;
  const bool fused = e.cfg.precision == BM_PREC_BF16;
  const unsigned long long sig_value = t != nullptr ? t->seq + 1 : 0;  // this task's completion
  if (signal != nullptr && t != nullptr) signal += t->seq % kSignalSlots;  // its own slot
  const int L = lstm ? c.d.layers : 1;
  for (int l = 0; l < L; ++l) {
    const bool last = l == L - 1 && !proj;
    bm_status s = launch_one_step(e, c, rows_dev, rows_host, b, l, false, (last && fused) ? signal : nullptr,
                                  sig_value);
    if (s != BM_OK) return s;
  }
  if (proj) {
    bm_status s = launch_one_step(e, c, rows_dev, rows_host, b, 0, true, fused ? signal : nullptr, sig_value);
    if (s != BM_OK) return s;
  }
  if (signal != nullptr && !fused) {
    CK(launch_signal(signal, sig_value, e.stream));
    e.stats.kernel_launches += 1;
  }
  return BM_OK;
}

bm_status launch_tasks(Engine& e, std::vector<Task>& tasks) {
  if (tasks.empty()) return BM_OK;
  int total = 0;
  for (Task& t : tasks) total += static_cast<int>(t.rows.size());
  for (Task& t : tasks) {
    t.seq = e.launched++;
    t.b = static_cast<int>(t.rows.size());
    e.stats.tasks += 1;
    e.stats.rows += t.b;
    if (e.cfg.clock != BM_CLOCK_WALL) {
      const double start = std::max(e.now, e.last_finish);
      t.finish = start + 1.0;
      e.last_finish = t.finish;
    }
    const uint64_t task_index = e.tasks_total++;
    if (e.cfg.record_log) {
      bm_task_record rec;
      rec.task = static_cast<int>(task_index);
      rec.worker = e.cur;
      rec.cell = t.ct;
      rec.tick = t.tick;
      rec.first_row = static_cast<int>(e.log_rows.size());
      rec.n_rows = t.b;
      e.log_tasks.push_back(rec);
      for (const TaskRow& tr : t.rows) e.log_rows.push_back({e.reqs[tr.req].id, tr.node, tr.slot});
    }
  }
  if (!e.device()) return BM_OK;
  static const int rows_inline = getenv("BM_ROWS_INLINE") ? atoi(getenv("BM_ROWS_INLINE")) : 0;
  if (e.cfg.precision == BM_PREC_BF16 && !e.persistent_active && rows_inline) {
    // diagnostics: each launch carries its task's row descriptors as a kernel parameter
    for (Task& t : tasks) {
      bm_status s = launch_cell(e, e.cells[t.ct], nullptr, t.desc.data(), t.b, &t, e.signal_dev);
      if (s != BM_OK) return s;
    }
    return BM_OK;
  }
  // ring placement: one contiguous region for all tasks of this Schedule call
  if (total > e.ring_rows) return BM_E_INVAL;
  if (e.ring_head + total > e.ring_rows) e.ring_head = 0;
  const int base = e.ring_head;
  int off = base;
  for (Task& t : tasks) {
    t.ring_off = off;
    memcpy(e.ring_host + off, t.desc.data(), sizeof(RowDesc) * t.b);
    off += t.b;
  }
  e.ring_head = off;
  if (e.persistent_active) {
    // rows first, then the headers that publish them (same copy stream: ordered)
    CK(cudaMemcpyAsync(e.ring_dev + base, e.ring_host + base, sizeof(RowDesc) * total,
                       cudaMemcpyHostToDevice, e.copy_stream));
    const int n = static_cast<int>(tasks.size());
    const int h0 = static_cast<int>((tasks[0].seq - e.run_base) % e.hdr_ring);
    for (int i = 0; i < n; ++i) {
      Task& t = tasks[i];
      TaskHdr& h = e.hdr_host[(h0 + i) % e.hdr_ring];
      h.seq = static_cast<int32_t>(t.seq - e.run_base);
      h.b = t.b;
      h.row_off = t.ring_off;
      h.flags = 0;
      if (e.cfg.time_kernels) {
        double bytes, flops;
        algo_cost(e, e.cells[t.ct], t.b, false, &bytes, &flops);
        account_launch(e, BM_K_PERSISTENT, t.b, bytes, flops);
      }
    }
    const int first = std::min(n, e.hdr_ring - h0);
    CK(cudaMemcpyAsync(e.hdr_dev + h0, e.hdr_host + h0, sizeof(TaskHdr) * first, cudaMemcpyHostToDevice,
                       e.copy_stream));
    if (first < n)
      CK(cudaMemcpyAsync(e.hdr_dev, e.hdr_host, sizeof(TaskHdr) * (n - first), cudaMemcpyHostToDevice,
                         e.copy_stream));
    return BM_OK;
  }
  // descriptors travel on the copy stream: the copy overlaps the kernels still running
  CK(cudaMemcpyAsync(e.ring_dev + base, e.ring_host + base, sizeof(RowDesc) * total,
                     cudaMemcpyHostToDevice, e.copy_stream));
  if (e.cfg.precision == BM_PREC_BF16) {
    // tcgen05 path: publish the rows with a flag write behind the copy; each launch polls the
    // flag on the device, so the kernel stream never waits on the copy stream (PDL stays on)
    const unsigned int seq = ++e.rows_seq;
    if (e.write_value32 != nullptr) {
      using WV = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
      if (reinterpret_cast<WV>(e.write_value32)(e.copy_stream, reinterpret_cast<CUdeviceptr>(e.rows_flag_dev),
                                                seq, 0) != CUDA_SUCCESS)
        return BM_E_CUDA;
    } else {
      unsigned int* v = e.rows_seq_host + (seq % 256);
      *v = seq;
      CK(cudaMemcpyAsync(e.rows_flag_dev, v, 4, cudaMemcpyHostToDevice, e.copy_stream));
    }
    e.launch_rows_seq = seq;
    for (Task& t : tasks) {
      bm_status s = launch_cell(e, e.cells[t.ct], e.ring_dev + t.ring_off, nullptr, t.b, &t, e.signal_dev);
      if (s != BM_OK) {
        e.launch_rows_seq = 0;
        return s;
      }
    }
    e.launch_rows_seq = 0;
    return BM_OK;
  }
  CK(cudaEventRecord(e.copy_ev, e.copy_stream));
  CK(cudaStreamWaitEvent(e.stream, e.copy_ev, 0));
  for (Task& t : tasks) {
    bm_status s = launch_cell(e, e.cells[t.ct], e.ring_dev + t.ring_off, nullptr, t.b, &t, e.signal_dev);
    if (s != BM_OK) return s;
  }
  return BM_OK;
}

// While a task's completion slot has not landed, the spin loops query the stream every 4096
// polls (~0.5 ms): a CUDA error (a fault, or a kernel's 10 s dependency-wait trap) makes the
// engine sticky (BM_E_CUDA, include/bm.h); so does an idle stream whose task never signalled
// (e.g. the persistent kernel aborted), instead of spinning forever.
static bool completion_lost(Engine& e, volatile unsigned long long* sig, uint64_t seq) {
  const cudaError_t q = cudaStreamQuery(e.stream);
  if (q == cudaErrorNotReady) return false;
  if (q == cudaSuccess && *sig > seq) return false;  // landed meanwhile
  if (!e.sticky_cuda)
    fprintf(stderr, "bm: task %llu never signalled completion (%s)\n", static_cast<unsigned long long>(seq),
            q == cudaSuccess ? "stream idle" : cudaGetErrorString(q));
  e.sticky_cuda = true;
  return true;
}

// Retire the active worker's oldest in-flight task if the device has finished it (and, on the
// virtual clock, its tick has come). Returns 1 if retired, 0 if not (yet), -1 on a CUDA error.
static int retire_front(Engine& e, bool block) {
  if (e.inflight.empty()) return 0;
  Task& t = e.inflight.front();
  if (e.cfg.clock != BM_CLOCK_WALL && t.finish > e.now) return 0;
  if (e.device()) {
    // the task's own signal slot (kSignalSlots-entry ring, written once per task)
    volatile unsigned long long* sig = e.signal_host + (t.seq % kSignalSlots);
    if (*sig <= t.seq) {
      if (!block && e.cfg.clock == BM_CLOCK_WALL) {
        if ((++e.poll_spins & 4095) == 0 && completion_lost(e, sig, t.seq)) return -1;
        return 0;
      }
      for (uint64_t it = 1; *sig <= t.seq; ++it)
        if ((it & 4095) == 0 && completion_lost(e, sig, t.seq)) return -1;
    }
  }
  if (e.tl_dev != nullptr && t.seq < Engine::kTimeline) e.tl_retire[t.seq] = realtime_ns();
  if (e.cfg.clock == BM_CLOCK_WALL) e.now = wall_now(e);
  const auto t0 = std::chrono::steady_clock::now();
  retire_task(e, t);
  e.inflight.pop_front();
  e.stats.retire_ns += std::chrono::duration<double, std::nano>(std::chrono::steady_clock::now() - t0).count();
  return 1;
}

// Retire every finished in-flight task of every worker. Virtual clock: in (finish tick,
// worker) order (S21 with W workers, as the replay); wall clock: each worker's FIFO.
static bm_status retire_ready(Engine& e, bool block) {
  const int W = e.cfg.workers;
  int r = 0;
  if (W == 1) {
    while ((r = retire_front(e, block)) > 0) {
    }
    return r < 0 ? BM_E_CUDA : BM_OK;
  }
  if (e.cfg.clock != BM_CLOCK_WALL) {
    for (;;) {
      int best = -1;
      double bf = 0;
      for (int w = 0; w < W; ++w) {
        const std::deque<Task>& q = e.inflight_of(w);
        if (!q.empty() && q.front().finish <= e.now && (best < 0 || q.front().finish < bf)) {
          best = w;
          bf = q.front().finish;
        }
      }
      if (best < 0) break;
      select_worker(e, best);
      if ((r = retire_front(e, block)) < 0) return BM_E_CUDA;
    }
  } else {
    for (int w = 0; w < W; ++w) {
      select_worker(e, w);
      while ((r = retire_front(e, block)) > 0) {
      }
      if (r < 0) return BM_E_CUDA;
    }
  }
  return BM_OK;
}

static void admit_due(Engine& e) {
  while (!e.pending.empty() && e.reqs[e.pending.front()].t_arrival <= e.now) {
    const int ri = e.pending.front();
    e.pending.pop_front();
    admit_request(e, ri);
  }
}

static bm_status schedule_and_launch_one(Engine& e, int* n_tasks);

// Schedule(worker) for every idle worker, in id order (Alg. 1: "whenever some worker becomes
// idle", L371; S19 idle = <= k outstanding tasks).
static bm_status schedule_and_launch(Engine& e, int* n_tasks) {
  *n_tasks = 0;
  for (int w = 0; w < e.cfg.workers; ++w) {
    select_worker(e, w);
    int n = 0;
    bm_status s = schedule_and_launch_one(e, &n);
    if (s != BM_OK) return s;
    *n_tasks += n;
  }
  return BM_OK;
}

static bm_status schedule_and_launch_one(Engine& e, int* n_tasks) {
  *n_tasks = 0;
  if (static_cast<int>(e.inflight.size()) > e.cfg.schedule_when_outstanding_leq) return BM_OK;
  static thread_local std::vector<Task> tasks;
  tasks.clear();
  const auto t0 = std::chrono::steady_clock::now();
  schedule(e, e.cur, tasks);
  e.stats.sched_ns += std::chrono::duration<double, std::nano>(std::chrono::steady_clock::now() - t0).count();
  e.stats.schedule_calls += 1;
  if (tasks.empty()) return BM_OK;
  const auto t1 = std::chrono::steady_clock::now();
  bm_status s = migrate_inputs(e, tasks);
  if (s == BM_OK) s = launch_tasks(e, tasks);
  e.stats.launch_ns += std::chrono::duration<double, std::nano>(std::chrono::steady_clock::now() - t1).count();
  if (s != BM_OK) return s;
  for (Task& t : tasks) e.inflight.push_back(std::move(t));
  *n_tasks = static_cast<int>(tasks.size());
  return BM_OK;
}

static bool all_done(Engine& e) {
  for (int w = 0; w < e.cfg.workers; ++w)
    if (!e.inflight_of(w).empty()) return false;
  return e.pending.empty() && !has_ready(e);
}

// One round of the virtual-time event loop (S21); advances the clock to the next event.
static bm_status virtual_round(Engine& e, int* n_tasks) {
  *n_tasks = 0;
  if (retire_ready(e, true) != BM_OK) return BM_E_CUDA;
  admit_due(e);
  bm_status s = schedule_and_launch(e, n_tasks);
  if (s != BM_OK) return s;
  double next = 1e300;
  for (int w = 0; w < e.cfg.workers; ++w)
    if (!e.inflight_of(w).empty()) next = std::min(next, e.inflight_of(w).front().finish);
  if (!e.pending.empty()) next = std::min(next, e.reqs[e.pending.front()].t_arrival);
  if (next == 1e300) return all_done(e) ? BM_E_AGAIN : BM_E_STATE;  // nothing can progress
  e.now = next;
  return BM_OK;
}

}  // namespace bm

using namespace bm;

// ================================================================= C-ABI
extern "C" {

int bm_abi_version(void) { return BM_ABI_VERSION; }

const char* bm_strerror(bm_status s) {
  switch (s) {
    case BM_OK: return "ok";
    case BM_E_INVAL: return "invalid argument";
    case BM_E_NOMEM: return "out of memory";
    case BM_E_FULL: return "request table full";
    case BM_E_AGAIN: return "nothing to do";
    case BM_E_CUDA: return "CUDA error (sticky)";
    case BM_E_STATE: return "invalid state";
    case BM_E_NODEV: return "no sm_100 device";
  }
  return "unknown";
}

void bm_config_default(bm_config* c) {
  memset(c, 0, sizeof(*c));
  c->device = 0;
  c->precision = BM_PREC_BF16;
  c->clock = BM_CLOCK_WALL;
  c->hidden = 1024;
  c->pool_layers = 1;
  c->max_slots = 65536;
  c->max_requests = 65536;
  c->max_tasks_to_submit = 5;
  c->min_followon_batch = 1;
  c->schedule_when_outstanding_leq = 0;
  c->max_decode_len = 512;
  c->keep_results = 0;
  c->record_logits = 0;
  c->time_kernels = 0;
  c->record_log = 1;
  c->persistent = 0;
  c->policy = BM_POLICY_CELLULAR;
  c->bucket_width = 10;
  c->workers = 1;
  c->devices = 1;
}

static void dump_timeline(Engine& e) {
  const char* path = getenv("BM_TIMELINE");
  if (path == nullptr || e.tl_dev == nullptr || cudaStreamSynchronize(e.stream) != cudaSuccess) return;
  std::vector<unsigned long long> d(4 * Engine::kTimeline);
  if (cudaMemcpy(d.data(), e.tl_dev, d.size() * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return;
  FILE* f = fopen(path, "a");
  if (f == nullptr) return;
  fprintf(f, "# launch b host_issue_ns dev_start_ns dev_wait_ns dev_end_ns ctas\n");
  for (uint64_t i = 0; i < e.tl_n; ++i)
    fprintf(f, "L %llu %d %lld %llu %llu %llu %llu\n", static_cast<unsigned long long>(i), e.tl_b[i],
            e.tl_host[i], ~d[4 * i], ~d[4 * i + 1], d[4 * i + 2], d[4 * i + 3]);
  for (uint64_t i = 0; i < std::min<uint64_t>(e.launched, Engine::kTimeline); ++i)
    if (e.tl_retire[i]) fprintf(f, "R %llu %lld\n", static_cast<unsigned long long>(i), e.tl_retire[i]);
  fclose(f);
}

static void free_device(Engine& e) {
  select_worker(e, 0);
  for (size_t ci = 1; ci < e.ctxs.size(); ++ci) {
    DevCtx& x = e.ctxs[ci];
    if (!e.device()) break;
    cudaSetDevice(x.cuda_dev);
    cudaFree(x.h_pool);
    cudaFree(x.c_pool);
    cudaFree(x.tok);
    cudaFree(x.dead);
    cudaFree(x.ring_dev);
    cudaFree(x.rows_flag_dev);
    if (x.ring_host) cudaFreeHost(x.ring_host);
    if (x.rows_seq_host) cudaFreeHost(x.rows_seq_host);
    if (x.copy_stream) cudaStreamDestroy(x.copy_stream);
    if (x.copy_ev) cudaEventDestroy(x.copy_ev);
    for (CellWeights& w : x.cells) {
      for (void* p : w.W) cudaFree(p);
      for (float* p : w.bias) cudaFree(p);
      cudaFree(w.E);
      cudaFree(w.W_out);
      cudaFree(w.b_out);
    }
  }
  if (e.device() && e.ctxs.size() > 1) cudaSetDevice(e.ctxs[0].cuda_dev);
  for (size_t w = 1; w < e.parked.size(); ++w) {
    WorkerState& ws = e.parked[w];
    if (ws.stream) {
      cudaStreamSynchronize(ws.stream);
      cudaStreamDestroy(ws.stream);
    }
    if (ws.signal_host) cudaFreeHost(ws.signal_host);
    cudaFree(ws.dep_flag);
    cudaFree(ws.sig_ctas);
    cudaFree(ws.done_ctas);
    cudaFree(ws.amax);
    cudaFree(ws.scratch);
  }
  if (!e.device()) return;
  dump_timeline(e);
  cudaFree(e.tl_dev);
  for (Cell& c : e.cells) {
    for (void* p : c.W) cudaFree(p);
    for (float* p : c.bias) cudaFree(p);
    cudaFree(c.E);
    cudaFree(c.W_out);
    cudaFree(c.b_out);
  }
  cudaFree(e.h_pool);
  cudaFree(e.c_pool);
  cudaFree(e.tok);
  cudaFree(e.dead);
  if (e.eos_host) cudaFreeHost(e.eos_host);
  cudaFree(e.res_h);
  cudaFree(e.res_c);
  cudaFree(e.res_tok);
  cudaFree(e.logits);
  cudaFree(e.amax);
  cudaFree(e.scratch);
  cudaFree(e.done_ctas);
  cudaFree(e.sig_ctas);
  cudaFree(e.dep_flag);
  cudaFree(e.ring_dev);
  cudaFree(e.direct_rows);
  cudaFree(e.phase_dev);
  if (e.direct_host) cudaFreeHost(e.direct_host);
  for (cudaEvent_t ev : e.direct_ev)
    if (ev) cudaEventDestroy(ev);
  if (e.ring_host) cudaFreeHost(e.ring_host);
  if (e.signal_host) cudaFreeHost(e.signal_host);
  cudaFree(e.spans);
  cudaFree(e.span_log);
  if (e.copy_stream) cudaStreamDestroy(e.copy_stream);
  if (e.copy_ev) cudaEventDestroy(e.copy_ev);
  cudaFree(e.hdr_dev);
  if (e.hdr_host) cudaFreeHost(e.hdr_host);
  cudaFree(e.gbar);
  cudaFree(e.perr);
  cudaFree(e.rows_flag_dev);
  if (e.rows_seq_host) cudaFreeHost(e.rows_seq_host);
  if (e.stream) cudaStreamDestroy(e.stream);
}

bm_status bm_create(const bm_config* cfg, bm_engine** out) {
  if (cfg == nullptr || out == nullptr) return BM_E_INVAL;
  const bm_config& c = *cfg;
  if (c.hidden <= 0 || c.hidden % 64 != 0 || c.pool_layers < 1 || c.pool_layers > 8 ||
      c.max_slots < 1 || c.max_requests < 1 || c.max_requests >= (1 << 23) ||
      c.max_tasks_to_submit < 1 || c.min_followon_batch < 1 || c.schedule_when_outstanding_leq < 0 ||
      c.max_decode_len < 1 || c.precision < 0 || c.precision > 1 || c.clock < 0 || c.clock > 2 ||
      c.policy < 0 || c.policy > 1 || c.bucket_width < 1 || c.workers < 1 || c.workers > 8 ||
      c.devices < 1 || c.devices > c.workers || (c.devices > 1 && c.persistent) ||
      (c.workers > 1 && c.policy != BM_POLICY_CELLULAR) ||
      // tasks in flight per worker (<= k + MaxTasksToSubmit) must fit the completion-signal
      // ring and the persistent kernel's task-header ring (both kSignalSlots = 256 entries)
      c.max_tasks_to_submit + c.schedule_when_outstanding_leq + 2 > kSignalSlots)
    return BM_E_INVAL;
  Engine* e = new (std::nothrow) Engine();
  if (e == nullptr) return BM_E_NOMEM;
  e->cfg = c;
  e->reqs.resize(c.max_requests);
  e->free_slots_heap.resize(c.max_slots);
  for (int i = 0; i < c.max_slots; ++i) e->free_slots_heap[i] = i;  // sorted == valid min-heap
  e->t0 = std::chrono::steady_clock::now();
  if (c.workers > 1) e->parked.resize(c.workers);
  // device contexts (§8f N2): worker w on context w % devices; every slot starts nowhere
  e->ctxs.resize(c.devices);
  e->worker_ctx.resize(c.workers);
  for (int w = 0; w < c.workers; ++w) e->worker_ctx[w] = w % c.devices;
  e->slot_ctx.assign(c.max_slots, -1);
  if (e->device()) {
    Engine& E = *e;
    auto fail = [&](bm_status s) {
      free_device(E);
      delete e;
      return s;
    };
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= c.device) return fail(BM_E_NODEV);
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, c.device) != cudaSuccess || prop.major != 10)
      return fail(BM_E_NODEV);
    if (cudaSetDevice(c.device) != cudaSuccess) return fail(BM_E_NODEV);
    if (cudaStreamCreateWithFlags(&E.stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&E.copy_stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&E.copy_ev, cudaEventDisableTiming) != cudaSuccess)
      return fail(BM_E_CUDA);
    const size_t H = c.hidden, S = c.max_slots, L = c.pool_layers, R = c.max_requests;
    const size_t el = E.elem();
    bool ok = cudaMalloc(&E.h_pool, L * 2 * S * H * el) == cudaSuccess &&
              dalloc(&E.c_pool, L * S * H) == cudaSuccess && dalloc(&E.tok, S) == cudaSuccess &&
              dalloc(&E.dead, S) == cudaSuccess &&
              dalloc(&E.res_h, R * L * H) == cudaSuccess && dalloc(&E.res_c, R * L * H) == cudaSuccess &&
              dalloc(&E.res_tok, R * static_cast<size_t>(c.max_decode_len)) == cudaSuccess &&
              dalloc(&E.amax, 512) == cudaSuccess && dalloc(&E.done_ctas, 1) == cudaSuccess &&
              dalloc(&E.sig_ctas, 1) == cudaSuccess && dalloc(&E.dep_flag, 1) == cudaSuccess &&
              dalloc(&E.direct_rows, 2 * 4096) == cudaSuccess &&
              cudaEventCreateWithFlags(&E.direct_ev[0], cudaEventDisableTiming) == cudaSuccess &&
              cudaEventCreateWithFlags(&E.direct_ev[1], cudaEventDisableTiming) == cudaSuccess;
    if (ok && c.precision == BM_PREC_BF16)  // cell_pair2_kernel's split-K exchange regions
      ok = dalloc(&E.scratch, static_cast<size_t>(kPairScratchCTAs) * 128 * 256) == cudaSuccess;
    if (!ok) return fail(BM_E_NOMEM);
    // descriptor ring: every worker keeps <= k + MaxTasksToSubmit tasks of <= 512 rows in
    // flight, and a Schedule call's rows are placed contiguously (a wrap wastes the tail):
    // twice that bound, so rows of a task still in flight are never overwritten
    E.ring_rows = std::max(64, c.workers * (c.max_tasks_to_submit + c.schedule_when_outstanding_leq + 2)) * 512 * 2;
    if (dalloc(&E.ring_dev, E.ring_rows) != cudaSuccess) return fail(BM_E_NOMEM);
    if (cudaHostAlloc(reinterpret_cast<void**>(&E.ring_host), E.ring_rows * sizeof(RowDesc),
                      cudaHostAllocDefault) != cudaSuccess)
      return fail(BM_E_NOMEM);
    if (cudaHostAlloc(reinterpret_cast<void**>(&E.signal_host), kSignalSlots * sizeof(unsigned long long),
                      cudaHostAllocMapped) != cudaSuccess)
      return fail(BM_E_NOMEM);
    memset(E.signal_host, 0, kSignalSlots * sizeof(unsigned long long));
    // <eos> reports (N1): written by the projection kernel, read at retire
    if (cudaHostAlloc(reinterpret_cast<void**>(&E.eos_host), R * sizeof(int), cudaHostAllocMapped) != cudaSuccess ||
        cudaHostGetDevicePointer(reinterpret_cast<void**>(&E.eos_dev), E.eos_host, 0) != cudaSuccess)
      return fail(BM_E_NOMEM);
    memset(E.eos_host, 0, R * sizeof(int));
    // ring-row publication flag (device) + the stream-write entry point (or a pinned value ring)
    if (dalloc(&E.rows_flag_dev, 1) != cudaSuccess ||
        cudaHostAlloc(reinterpret_cast<void**>(&E.rows_seq_host), 256 * sizeof(unsigned int),
                      cudaHostAllocDefault) != cudaSuccess)
      return fail(BM_E_NOMEM);
    {
      cudaDriverEntryPointQueryResult q;
      void* fn = nullptr;
      if (!getenv("BM_NO_WRITE_VALUE") &&
          cudaGetDriverEntryPoint("cuStreamWriteValue32", &fn, cudaEnableDefault, &q) == cudaSuccess &&
          q == cudaDriverEntryPointSuccess)
        E.write_value32 = fn;
    }
    if (cudaHostGetDevicePointer(reinterpret_cast<void**>(&E.signal_dev), E.signal_host, 0) != cudaSuccess)
      return fail(BM_E_CUDA);
    if (cudaMemsetAsync(E.h_pool, 0, L * 2 * S * H * el, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.c_pool, 0, L * S * H * 4, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.tok, 0, S * 4, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.dead, 0, S * 4, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.amax, 0, 512 * 8, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.done_ctas, 0, 4, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.sig_ctas, 0, 4, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.dep_flag, 0, 4, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.rows_flag_dev, 0, 4, E.stream) != cudaSuccess ||
        cudaMemsetAsync(E.res_tok, 0, R * c.max_decode_len * 4, E.stream) != cudaSuccess)
      return fail(BM_E_CUDA);
    if (c.time_kernels) {
      // device-side launch spans: 64 slots {start, ctas}, per-class accumulators {ns, launches},
      // and the per-launch span log
      if (dalloc(&E.spans, 2 * 64 + 2 * BM_K_CLASSES) != cudaSuccess ||
          dalloc(&E.span_log, Engine::kLaunchLog) != cudaSuccess ||
          cudaMemsetAsync(E.spans, 0xFF, 2 * 64 * 8, E.stream) != cudaSuccess ||
          cudaMemsetAsync(E.span_log, 0, Engine::kLaunchLog * 8, E.stream) != cudaSuccess)
        return fail(BM_E_NOMEM);
      for (int i = 0; i < 64; ++i)
        if (cudaMemsetAsync(E.spans + 2 * i + 1, 0, 8, E.stream) != cudaSuccess) return fail(BM_E_CUDA);
      if (cudaMemsetAsync(E.spans + 128, 0, 16 * BM_K_CLASSES, E.stream) != cudaSuccess) return fail(BM_E_CUDA);
      E.launch_class.assign(Engine::kLaunchLog, 0);
      E.launch_b.assign(Engine::kLaunchLog, 0);
    }
    if (getenv("BM_TIMELINE") != nullptr) {
      if (dalloc(&E.tl_dev, 4 * Engine::kTimeline) != cudaSuccess ||
          cudaMemsetAsync(E.tl_dev, 0, 4 * Engine::kTimeline * 8, E.stream) != cudaSuccess)
        return fail(BM_E_NOMEM);
      E.tl_host.assign(Engine::kTimeline, 0);
      E.tl_retire.assign(Engine::kTimeline, 0);
      E.tl_b.assign(Engine::kTimeline, 0);
    }
    // device contexts 1..D-1 (§8f N2): CUDA device (device + c) % count, each with its own
    // state pool, descriptor ring and copy stream (the weight replicas follow in bm_load_cell);
    // peer access lets every context's kernels write the result rows on context 0
    for (int ci = 0; ci < c.devices; ++ci) E.ctxs[ci].cuda_dev = (c.device + ci) % ndev;
    for (int ci = 1; ci < c.devices; ++ci) {
      DevCtx& x = E.ctxs[ci];
      if (cudaSetDevice(x.cuda_dev) != cudaSuccess) return fail(BM_E_CUDA);
      if (x.cuda_dev != c.device) {
        cudaDeviceEnablePeerAccess(c.device, 0);
        cudaGetLastError();  // already enabled / unsupported: peer copies still work via the host
      }
      if (cudaMalloc(&x.h_pool, L * 2 * S * H * el) != cudaSuccess || dalloc(&x.c_pool, L * S * H) != cudaSuccess ||
          dalloc(&x.tok, S) != cudaSuccess || dalloc(&x.dead, S) != cudaSuccess ||
          dalloc(&x.ring_dev, E.ring_rows) != cudaSuccess || dalloc(&x.rows_flag_dev, 1) != cudaSuccess ||
          cudaHostAlloc(reinterpret_cast<void**>(&x.ring_host), E.ring_rows * sizeof(RowDesc), cudaHostAllocDefault) !=
              cudaSuccess ||
          cudaHostAlloc(reinterpret_cast<void**>(&x.rows_seq_host), 256 * sizeof(unsigned int), cudaHostAllocDefault) !=
              cudaSuccess ||
          cudaStreamCreateWithFlags(&x.copy_stream, cudaStreamNonBlocking) != cudaSuccess ||
          cudaEventCreateWithFlags(&x.copy_ev, cudaEventDisableTiming) != cudaSuccess)
        return fail(BM_E_NOMEM);
      if (cudaMemset(x.h_pool, 0, L * 2 * S * H * el) != cudaSuccess || cudaMemset(x.c_pool, 0, L * S * H * 4) != cudaSuccess ||
          cudaMemset(x.tok, 0, S * 4) != cudaSuccess || cudaMemset(x.dead, 0, S * 4) != cudaSuccess ||
          cudaMemset(x.rows_flag_dev, 0, 4) != cudaSuccess)
        return fail(BM_E_CUDA);
    }
    if (c.devices > 1) {
      cudaSetDevice(c.device);
      for (int ci = 1; ci < c.devices; ++ci)
        if (E.ctxs[ci].cuda_dev != c.device) {
          cudaDeviceEnablePeerAccess(E.ctxs[ci].cuda_dev, 0);
          cudaGetLastError();
        }
    }
    // workers 1..W-1 (§8f N2): own stream, completion counter, launch chain, device scratch,
    // allocated on the worker's context device
    for (int w = 1; w < c.workers; ++w) {
      WorkerState& ws = E.parked[w];
      if (cudaSetDevice(E.ctxs[E.worker_ctx[w]].cuda_dev) != cudaSuccess) return fail(BM_E_CUDA);
      if (cudaStreamCreateWithFlags(&ws.stream, cudaStreamNonBlocking) != cudaSuccess ||
          cudaHostAlloc(reinterpret_cast<void**>(&ws.signal_host), kSignalSlots * sizeof(unsigned long long),
                        cudaHostAllocMapped) != cudaSuccess)
        return fail(BM_E_NOMEM);
      memset(ws.signal_host, 0, kSignalSlots * sizeof(unsigned long long));
      if (cudaHostGetDevicePointer(reinterpret_cast<void**>(&ws.signal_dev), ws.signal_host, 0) != cudaSuccess ||
          dalloc(&ws.dep_flag, 1) != cudaSuccess || dalloc(&ws.sig_ctas, 1) != cudaSuccess ||
          dalloc(&ws.done_ctas, 1) != cudaSuccess || dalloc(&ws.amax, 512) != cudaSuccess ||
          (c.precision == BM_PREC_BF16 &&
           dalloc(&ws.scratch, static_cast<size_t>(kPairScratchCTAs) * 128 * 256) != cudaSuccess))
        return fail(BM_E_NOMEM);
      if (cudaMemset(ws.dep_flag, 0, 4) != cudaSuccess || cudaMemset(ws.sig_ctas, 0, 4) != cudaSuccess ||
          cudaMemset(ws.done_ctas, 0, 4) != cudaSuccess || cudaMemset(ws.amax, 0, 512 * 8) != cudaSuccess)
        return fail(BM_E_CUDA);
    }
    cudaSetDevice(c.device);
    if (cudaStreamSynchronize(E.stream) != cudaSuccess) return fail(BM_E_CUDA);
  }
  *out = reinterpret_cast<bm_engine*>(e);
  return BM_OK;
}

void bm_destroy(bm_engine* h) {
  if (h == nullptr) return;
  Engine* e = reinterpret_cast<Engine*>(h);
  if (e->device() && e->stream) cudaStreamSynchronize(e->stream);
  free_device(*e);
  delete e;
}

void* bm_stream(bm_engine* h) { return h ? reinterpret_cast<Engine*>(h)->stream : nullptr; }

bm_status bm_load_cell(bm_engine* h, const bm_cell_desc* d, const bm_weights* w, int* cell_id) {
  if (h == nullptr || d == nullptr || w == nullptr || cell_id == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  e.pdl_ok = false;  // other stream work follows: the next launch is fully ordered
  if (e.sticky_cuda) return BM_E_CUDA;
  if (e.submitted_any) return BM_E_STATE;
  if (e.cells.size() >= 64) return BM_E_INVAL;
  const int H = e.cfg.hidden;
  if (d->hidden != H || d->max_batch < 1 || d->max_batch > 512) return BM_E_INVAL;
  Cell c;
  c.d = *d;
  switch (d->kind) {
    case BM_CELL_LSTM:
    case BM_CELL_LSTM_PROJ:
      if (d->layers < 1 || d->layers > e.cfg.pool_layers || d->vocab < 1) return BM_E_INVAL;
      if (d->kind == BM_CELL_LSTM_PROJ && (d->vocab % 128 != 0 || w->W_out == nullptr || w->b_out == nullptr))
        return BM_E_INVAL;
      c.epi = EPI_LSTM, c.G = 4, c.U = 32, c.K0 = H, c.K1 = H;
      break;
    case BM_CELL_TREE_LEAF:
      if (d->layers != 1 || d->vocab < 1) return BM_E_INVAL;
      c.epi = EPI_LEAF, c.G = 3, c.U = 32, c.K0 = H, c.K1 = 0;
      break;
    case BM_CELL_TREE_INTERNAL:
      if (d->layers != 1) return BM_E_INVAL;
      c.epi = EPI_INTERNAL, c.G = 5, c.U = 16, c.K0 = H, c.K1 = H;
      break;
    default:
      return BM_E_INVAL;
  }
  const int K = c.K0 + c.K1;
  c.S = std::max(1, K / 512);          // fixed K slice of 512 -> batch-invariant reduction order
  // leaf cells (K = h): 256-wide slices (S = 4) so h/U x S = 128 CTAs stream the weights
  // instead of 64 (BM_LEAF_S=2 keeps the 512-wide slices)
  static const int env_leaf_s = getenv("BM_LEAF_S") ? atoi(getenv("BM_LEAF_S")) : 4;
  if (c.epi == EPI_LEAF && env_leaf_s == 4 && e.cfg.precision == BM_PREC_BF16 && K % 1024 == 0)
    c.S = std::min(4, K / 256);
  c.kslice = K / c.S;
  if (c.S > 8 || c.kslice % 64 != 0) return BM_E_INVAL;
  if (w->W == nullptr || w->b == nullptr) return BM_E_INVAL;
  const int L = (d->kind == BM_CELL_LSTM || d->kind == BM_CELL_LSTM_PROJ) ? d->layers : 1;
  for (int l = 0; l < L; ++l)
    if (w->W[l] == nullptr || w->b[l] == nullptr) return BM_E_INVAL;
  if (d->kind != BM_CELL_TREE_INTERNAL && w->E == nullptr) return BM_E_INVAL;
  if (e.device()) {
    const bool bf = e.cfg.precision == BM_PREC_BF16;
    const size_t el = e.elem();
    const size_t rows = static_cast<size_t>(c.G) * H;
    // every weight array may be a host pointer (copied up) or a device pointer on the engine's
    // device (adopted in place: the packing kernels read it directly, e.g. after an NCCL
    // broadcast). A device pointer of another device is rejected.
    auto on_device = [&](const void* p, bool* dev) -> bool {
      cudaPointerAttributes at{};
      if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        *dev = false;
        return true;
      }
      *dev = at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
      return !*dev || at.device == e.cfg.device;
    };
    std::vector<const void*> srcs;
    for (int l = 0; l < L; ++l) srcs.push_back(w->W[l]), srcs.push_back(w->b[l]);
    if (w->E != nullptr) srcs.push_back(w->E);
    if (d->kind == BM_CELL_LSTM_PROJ) srcs.push_back(w->W_out), srcs.push_back(w->b_out);
    for (const void* p : srcs) {
      bool dev;
      if (!on_device(p, &dev)) return BM_E_INVAL;
    }
    float* tmp = nullptr;
    float* tmpb = nullptr;
    const size_t maxsrc = std::max(rows * K, static_cast<size_t>(d->vocab) * H);
    CK(cudaMalloc(&tmp, maxsrc * 4));
    CK(cudaMalloc(&tmpb, std::max(rows, static_cast<size_t>(d->vocab)) * 4));
    // device source: use it as is; host source: copy into the staging buffer
    auto stage = [&](const float* src, float* buf, size_t n, const float** out) -> cudaError_t {
      bool dev = false;
      on_device(src, &dev);
      if (dev) {
        *out = src;
        return cudaSuccess;
      }
      *out = buf;
      return cudaMemcpyAsync(buf, src, n * 4, cudaMemcpyHostToDevice, e.stream);
    };
    const float* sw = nullptr;
    const float* sb = nullptr;
    for (int l = 0; l < L; ++l) {
      void* Wp = nullptr;
      float* bp = nullptr;
      CK(cudaMalloc(&Wp, rows * K * el));
      CK(dalloc(&bp, rows));
      CK(stage(w->W[l], tmp, rows * K, &sw));
      CK(stage(w->b[l], tmpb, rows, &sb));
      CK(launch_pack_rows(sw, Wp, bp, sb, c.G, H, K, bf ? 1 : 0, e.stream));
      if (bf)  // the tcgen05 kernel streams pre-swizzled stage tiles (overwrites the plain pack)
        CK(launch_pack_tiles(sw, Wp, c.G, H, K, c.G * c.U, static_cast<int>(rows), e.stream));
      CK(cudaStreamSynchronize(e.stream));
      c.W.push_back(Wp);
      c.bias.push_back(bp);
    }
    if (w->E != nullptr && d->kind != BM_CELL_TREE_INTERNAL) {
      const size_t n = static_cast<size_t>(d->vocab) * H;
      CK(cudaMalloc(&c.E, n * el));
      CK(stage(w->E, tmp, n, &sw));
      CK(launch_convert(sw, c.E, n, bf ? 1 : 0, e.stream));
      CK(cudaStreamSynchronize(e.stream));
    }
    if (d->kind == BM_CELL_LSTM_PROJ) {
      const size_t n = static_cast<size_t>(d->vocab) * H;
      CK(cudaMalloc(&c.W_out, n * el));
      CK(dalloc(&c.b_out, d->vocab));
      CK(stage(w->W_out, tmp, n, &sw));
      if (bf) CK(launch_pack_tiles(sw, c.W_out, 1, H, H, 128, d->vocab, e.stream));
      else CK(launch_convert(sw, c.W_out, n, 0, e.stream));
      CK(cudaMemcpyAsync(c.b_out, w->b_out, d->vocab * 4, cudaMemcpyDefault, e.stream));
      CK(cudaStreamSynchronize(e.stream));
      if (e.cfg.record_logits) {
        if (e.logits == nullptr) {
          CK(dalloc(&e.logits, static_cast<size_t>(e.cfg.max_requests) * e.cfg.max_decode_len * d->vocab));
          e.logits_vocab = d->vocab;
        } else if (e.logits_vocab != d->vocab) {
          return BM_E_INVAL;
        }
      }
    }
    cudaFree(tmp);
    cudaFree(tmpb);
    // weight replica on every other device context (§8f N2): the packed bytes, peer-copied
    for (size_t ci = 1; ci < e.ctxs.size(); ++ci) {
      DevCtx& x = e.ctxs[ci];
      CellWeights rep;
      const int dd = x.cuda_dev, sd = e.cfg.device;
      CK(cudaSetDevice(dd));
      auto clone = [&](const void* src, size_t bytes, void** dst) -> cudaError_t {
        *dst = nullptr;
        if (src == nullptr) return cudaSuccess;
        cudaError_t r = cudaMalloc(dst, bytes);
        return r != cudaSuccess ? r : cudaMemcpyPeer(*dst, dd, src, sd, bytes);
      };
      for (int l = 0; l < L; ++l) {
        void* wp = nullptr;
        void* bp = nullptr;
        CK(clone(c.W[l], rows * K * el, &wp));
        CK(clone(c.bias[l], rows * 4, &bp));
        rep.W.push_back(wp);
        rep.bias.push_back(static_cast<float*>(bp));
      }
      void* b_out = nullptr;
      CK(clone(c.E, static_cast<size_t>(d->vocab) * H * el, &rep.E));
      CK(clone(c.W_out, static_cast<size_t>(d->vocab) * H * el, &rep.W_out));
      CK(clone(c.b_out, static_cast<size_t>(d->vocab) * 4, &b_out));
      rep.b_out = static_cast<float*>(b_out);
      x.cells.resize(e.cells.size());
      x.cells.push_back(rep);
      CK(cudaSetDevice(sd));
    }
  }
  e.cells.push_back(c);
  for (size_t ci = 1; ci < e.ctxs.size(); ++ci) e.ctxs[ci].cells.resize(e.cells.size());
  *cell_id = static_cast<int>(e.cells.size()) - 1;
  return BM_OK;
}

static bool valid_tree(const bm_request* r) {
  const int n = r->n;
  if (n < 1 || r->left == nullptr || r->right == nullptr) return false;
  std::vector<int> parents(n, 0);
  for (int v = 0; v < n; ++v) {
    const int L = r->left[v], R = r->right[v];
    if ((L < 0) != (R < 0)) return false;       // binary: both children or none
    if (L >= 0) {
      if (L >= v || R >= v || L == R) return false;   // post-order: children first
      parents[L]++;
      parents[R]++;
    }
  }
  for (int v = 0; v < n - 1; ++v)
    if (parents[v] != 1) return false;
  return parents[n - 1] == 0;
}

bm_status bm_submit(bm_engine* h, const bm_request* q, uint64_t* req_id) {
  if (h == nullptr || q == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  if (e.sticky_cuda) return BM_E_CUDA;
  const int nc = static_cast<int>(e.cells.size());
  auto cell_ok = [&](int id, int k1, int k2) {
    return id >= 0 && id < nc && (e.cells[id].d.kind == k1 || e.cells[id].d.kind == k2);
  };
  if (q->n < 1 || q->tokens == nullptr) return BM_E_INVAL;
  if (e.cfg.policy == BM_POLICY_GRAPH && q->kind != BM_REQ_CHAIN) return BM_E_INVAL;  // [G5]
  int vocab = 0;
  if (q->kind == BM_REQ_CHAIN) {
    if (!cell_ok(q->cell0, BM_CELL_LSTM, BM_CELL_LSTM)) return BM_E_INVAL;
    vocab = e.cells[q->cell0].d.vocab;
  } else if (q->kind == BM_REQ_SEQ2SEQ) {
    if (!cell_ok(q->cell0, BM_CELL_LSTM, BM_CELL_LSTM) || !cell_ok(q->cell1, BM_CELL_LSTM_PROJ, BM_CELL_LSTM_PROJ))
      return BM_E_INVAL;
    if (q->decode_len < 1 || q->decode_len > e.cfg.max_decode_len) return BM_E_INVAL;
    if (e.cells[q->cell0].d.layers != e.cells[q->cell1].d.layers) return BM_E_INVAL;
    if (q->eos_stop && (q->eos_id < 0 || q->eos_id >= e.cells[q->cell1].d.vocab || q->decode_len > 4095))
      return BM_E_INVAL;
    vocab = e.cells[q->cell0].d.vocab;
  } else if (q->kind == BM_REQ_TREE) {
    if (!cell_ok(q->cell0, BM_CELL_TREE_LEAF, BM_CELL_TREE_LEAF) ||
        !cell_ok(q->cell1, BM_CELL_TREE_INTERNAL, BM_CELL_TREE_INTERNAL) || !valid_tree(q))
      return BM_E_INVAL;
    if (q->n > e.cfg.max_slots) return BM_E_INVAL;
    vocab = e.cells[q->cell0].d.vocab;
  } else {
    return BM_E_INVAL;
  }
  for (int i = 0; i < q->n; ++i) {
    const bool leaf_or_chain = q->kind != BM_REQ_TREE || q->left[i] < 0;
    if (leaf_or_chain && (q->tokens[i] < 0 || q->tokens[i] >= vocab)) return BM_E_INVAL;
  }
  // requests not yet admitted must arrive in submission order (an open-loop arrival stream;
  // each request is admitted at its own arrival, L323 / reading S21)
  if (!e.pending.empty() && q->arrival < e.reqs[e.pending.back()].t_arrival) return BM_E_INVAL;
  if (e.n_live_reqs >= e.cfg.max_requests) return BM_E_FULL;
  // request table slot: the entry of admission index id % max_requests must be free
  const int ri = static_cast<int>(e.next_req_id % e.cfg.max_requests);
  Request& r = e.reqs[ri];
  if (r.used) return BM_E_FULL;
  r.used = true;
  r.done = false;
  r.id = e.next_req_id++;
  r.tag = q->user_tag;
  r.kind = q->kind;
  r.cell0 = q->cell0;
  r.cell1 = q->cell1;
  r.t_arrival = q->arrival;
  r.tokens.assign(q->tokens, q->tokens + q->n);
  r.eos_stop = q->kind == BM_REQ_SEQ2SEQ && q->eos_stop != 0;
  r.eos_id = r.eos_stop ? q->eos_id : -1;
  r.dry_eos_step = r.eos_stop ? q->dry_eos_step : -1;
  r.decode_max = q->kind == BM_REQ_SEQ2SEQ ? q->decode_len : 0;
  if (q->kind == BM_REQ_CHAIN) {
    r.n_nodes = q->n;
    r.enc_len = q->n;
  } else if (q->kind == BM_REQ_SEQ2SEQ) {
    r.enc_len = q->n;
    r.n_nodes = q->n + q->decode_len;
  } else {
    r.n_nodes = q->n;
    r.left.assign(q->left, q->left + q->n);
    r.right.assign(q->right, q->right + q->n);
  }
  e.n_live_reqs += 1;
  e.submitted_any = true;
  e.pending.push_back(ri);
  if (req_id) *req_id = r.id;
  return BM_OK;
}

bm_status bm_submit_many(bm_engine* h, const bm_request* reqs, int n, uint64_t* first_id, int* n_done) {
  if (h == nullptr || reqs == nullptr || n < 0) return BM_E_INVAL;
  int k = 0;
  bm_status s = BM_OK;
  for (; k < n; ++k) {
    uint64_t id;
    s = bm_submit(h, reqs + k, &id);
    if (s != BM_OK) break;
    if (k == 0 && first_id) *first_id = id;
  }
  if (n_done) *n_done = k;
  return s;
}

bm_status bm_schedule_step(bm_engine* h, int* n_tasks) {
  if (h == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  if (e.sticky_cuda) return BM_E_CUDA;
  int n = 0;
  bm_status s;
  if (e.cfg.clock == BM_CLOCK_WALL) {
    if (!e.wall_started) {
      e.t0 = std::chrono::steady_clock::now();
      e.wall_started = true;
    }
    e.now = wall_now(e);
    s = retire_ready(e, false);
    if (s == BM_OK) {
      admit_due(e);
      s = schedule_and_launch(e, &n);
    }
    if (s == BM_OK && n == 0 && all_done(e)) s = BM_E_AGAIN;
  } else {
    s = virtual_round(e, &n);
  }
  select_worker(e, 0);
  if (n_tasks) *n_tasks = n;
  return s;
}

bm_status bm_poll(bm_engine* h, bm_completion* out, int cap, int* n) {
  if (h == nullptr || n == nullptr || (cap > 0 && out == nullptr)) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  if (e.cfg.clock == BM_CLOCK_WALL && e.device()) {
    e.now = wall_now(e);
    const bm_status s = retire_ready(e, false);
    select_worker(e, 0);
    if (s != BM_OK) return s;
  }
  const int k = std::min<int>(cap, static_cast<int>(e.completions.size()));
  if (k > 0) memcpy(out, e.completions.data(), k * sizeof(bm_completion));
  e.completions.erase(e.completions.begin(), e.completions.begin() + k);
  *n = k;
  return BM_OK;
}

static bool persistent_eligible(const Engine& e) {
  if (!e.cfg.persistent || !e.device() || e.cfg.precision != BM_PREC_BF16 || e.cells.size() != 1 ||
      e.cfg.workers != 1)
    return false;
  const Cell& c = e.cells[0];
  const int K = c.K0 + c.K1;
  return c.d.kind == BM_CELL_LSTM && c.d.layers == 1 && c.S >= 1 && c.S <= 4 && c.kslice <= 512 &&
         c.kslice % 64 == 0 && e.cfg.hidden % 32 == 0 && c.d.max_batch <= 512 && K == c.S * c.kslice;
}

static bm_status persistent_start(Engine& e) {
  e.pdl_ok = false;
  const Cell& c = e.cells[0];
  if (e.hdr_dev == nullptr) {
    CK(cudaMalloc(&e.hdr_dev, sizeof(TaskHdr) * e.hdr_ring));
    CK(cudaHostAlloc(reinterpret_cast<void**>(&e.hdr_host), sizeof(TaskHdr) * e.hdr_ring, cudaHostAllocDefault));
    CK(cudaMalloc(&e.gbar, sizeof(unsigned int)));
    CK(cudaMalloc(&e.perr, sizeof(int)));
  }
  CK(cudaStreamSynchronize(e.stream));
  CK(cudaMemsetAsync(e.hdr_dev, 0xFF, sizeof(TaskHdr) * e.hdr_ring, e.stream));  // seq = -1
  CK(cudaMemsetAsync(e.gbar, 0, sizeof(unsigned int), e.stream));
  CK(cudaMemsetAsync(e.perr, 0, sizeof(int), e.stream));
  PersistArgs a{};
  a.H = e.cfg.hidden;
  a.K = c.K0 + c.K1;
  a.K0 = c.K0;
  a.S = c.S;
  a.kslice = c.kslice;
  a.n_slots = e.cfg.max_slots;
  a.res_layers = e.cfg.pool_layers;
  a.hdr_ring = e.hdr_ring;
  a.hdr = e.hdr_dev;
  a.rows = e.ring_dev;
  a.E = c.E;
  a.h_pool = e.h_layer(0);
  a.c_pool = e.c_layer(0);
  a.tok = e.tok;
  a.W = c.W[0];
  a.bias = c.bias[0];
  a.res_h = e.res_h;
  a.res_c = e.res_c;
  a.gbar = e.gbar;
  a.err = e.perr;
  a.signal = e.signal_dev;
  a.sig_base = e.launched;  // == run_base below
  a.span = e.cfg.time_kernels ? e.spans : nullptr;
  a.span_acc = e.cfg.time_kernels ? e.spans + 128 + 2 * BM_K_PERSISTENT : nullptr;
  static const char* dump = getenv("BM_PHASE_DUMP");
  if (dump != nullptr && e.phase_dev == nullptr) CK(cudaMalloc(&e.phase_dev, 8 * 64 * 4096));
  if (e.phase_dev) CK(cudaMemsetAsync(e.phase_dev, 0, 8 * 64 * 4096, e.stream));
  a.phase = e.phase_dev;
  cudaError_t err = launch_lstm_persistent(a, e.stream);
  if (err == cudaErrorCooperativeLaunchTooLarge) {
    cudaGetLastError();
    return BM_E_AGAIN;  // cannot co-schedule every CTA: fall back to per-task launches
  }
  CK(err);
  e.persistent_active = true;
  e.run_base = e.launched;
  e.stats.kernel_launches += 1;
  return BM_OK;
}

static bm_status persistent_stop(Engine& e) {
  e.pdl_ok = false;
  if (!e.persistent_active) return BM_OK;
  const int idx = static_cast<int>((e.launched - e.run_base) % e.hdr_ring);
  // the slot's previous task retired long ago (at most k + MaxTasksToSubmit are in flight)
  TaskHdr& hd = e.hdr_host[idx];
  hd.seq = static_cast<int32_t>(e.launched - e.run_base);
  hd.b = -1;
  hd.row_off = 0;
  hd.flags = 0;
  CK(cudaMemcpyAsync(e.hdr_dev + idx, &hd, sizeof(TaskHdr), cudaMemcpyHostToDevice, e.copy_stream));
  CK(cudaStreamSynchronize(e.copy_stream));
  CK(cudaStreamSynchronize(e.stream));
  e.persistent_active = false;
  static const char* dump = getenv("BM_PHASE_DUMP");
  if (dump != nullptr && e.phase_dev != nullptr) {
    std::vector<unsigned long long> hh(16 * 4096);
    CK(cudaMemcpy(hh.data(), e.phase_dev, hh.size() * 8, cudaMemcpyDeviceToHost));
    FILE* f = fopen(dump, "a");
    if (f) {
      fprintf(f, "persistent task 20\n");
      for (int i = 0; i < 4096; ++i)
        if (hh[i * 16]) {
          fprintf(f, "%d", i);
          for (int k = 0; k < 16; ++k) fprintf(f, " %llu", hh[i * 16 + k]);
          fprintf(f, "\n");
        }
      fclose(f);
    }
  }
  int aborted = 0;
  CK(cudaMemcpy(&aborted, e.perr, sizeof(int), cudaMemcpyDeviceToHost));
  if (aborted) {
    e.sticky_cuda = true;
    return BM_E_CUDA;
  }
  return BM_OK;
}

bm_status bm_run(bm_engine* h, int* n_completed) {
  if (h == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::unique_lock<std::recursive_mutex> lk(e.mu);
  if (e.sticky_cuda) return BM_E_CUDA;
  const uint64_t before = e.completed_total;  // a concurrent bm_poll may drain e.completions
  int n = 0;
  bm_status s = BM_OK;
  if (persistent_eligible(e)) {
    s = persistent_start(e);
    if (s != BM_OK && s != BM_E_AGAIN) return s;
    s = BM_OK;
  }
  lk.unlock();
  if (e.cfg.clock == BM_CLOCK_WALL) {
    e.t0 = std::chrono::steady_clock::now();
    e.wall_started = true;
    while (true) {
      // one round of the event loop under the engine lock: a bm_poll on another thread
      // (the paper's poll thread, L395) interleaves between rounds
      std::lock_guard<std::recursive_mutex> round(e.mu);
      e.now = wall_now(e);
      s = retire_ready(e, false);
      if (s == BM_OK) {
        admit_due(e);
        s = schedule_and_launch(e, &n);
      }
      if (s != BM_OK) {
        select_worker(e, 0);
        persistent_stop(e);
        return s;
      }
      if (all_done(e)) break;
    }
  } else {
    for (;;) {
      std::lock_guard<std::recursive_mutex> round(e.mu);
      if ((s = virtual_round(e, &n)) != BM_OK) break;
    }
    if (s != BM_E_AGAIN) {
      std::lock_guard<std::recursive_mutex> g(e.mu);
      select_worker(e, 0);
      persistent_stop(e);
      return s;
    }
  }
  lk.lock();
  if (e.persistent_active) {
    s = persistent_stop(e);
    if (s != BM_OK) return s;
  }
  if (e.device()) {
    for (int w = e.cfg.workers - 1; w >= 0; --w) {
      select_worker(e, w);
      CK(cudaStreamSynchronize(e.stream));
    }
  }
  select_worker(e, 0);
  if (n_completed) *n_completed = static_cast<int>(e.completed_total - before);
  return BM_OK;
}

bm_status bm_read_result(bm_engine* h, uint64_t req_id, bm_result* dst) {
  if (h == nullptr || dst == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  e.pdl_ok = false;  // other stream work follows: the next launch is fully ordered
  if (e.sticky_cuda) return BM_E_CUDA;
  Request& r = e.reqs[req_id % e.cfg.max_requests];
  if (!r.used || r.id != req_id) return BM_E_INVAL;
  if (!r.done) return BM_E_STATE;
  if (!e.device()) return BM_E_STATE;
  const int ri = static_cast<int>(req_id % e.cfg.max_requests);
  const size_t H = e.H(), L = e.cfg.pool_layers;
  CK(cudaStreamSynchronize(e.stream));
  if (dst->h) CK(cudaMemcpyAsync(dst->h, e.res_h + ri * L * H, L * H * 4, cudaMemcpyDeviceToHost, e.stream));
  if (dst->c) CK(cudaMemcpyAsync(dst->c, e.res_c + ri * L * H, L * H * 4, cudaMemcpyDeviceToHost, e.stream));
  if (r.kind == BM_REQ_SEQ2SEQ) {
    // emitted tokens: up to and including the <eos> step under eos_stop (N1), else all steps
    const int T = r.eos_step >= 0 ? r.eos_step + 1 : r.n_nodes - r.enc_len;
    if (dst->tokens) {
      CK(cudaMemcpyAsync(dst->tokens, e.res_tok + static_cast<size_t>(ri) * e.cfg.max_decode_len, T * 4,
                         cudaMemcpyDeviceToHost, e.stream));
      CK(cudaStreamSynchronize(e.stream));
      for (int s = T; s < r.decode_max; ++s) dst->tokens[s] = -1;
    }
    if (dst->logits && e.logits)
      CK(cudaMemcpyAsync(dst->logits, e.logits + static_cast<size_t>(ri) * e.cfg.max_decode_len * e.logits_vocab,
                         static_cast<size_t>(T) * e.logits_vocab * 4, cudaMemcpyDeviceToHost, e.stream));
  }
  CK(cudaStreamSynchronize(e.stream));
  return BM_OK;
}

bm_status bm_release(bm_engine* h, uint64_t req_id) {
  if (h == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  Request& r = e.reqs[req_id % e.cfg.max_requests];
  if (!r.used || r.id != req_id) return BM_E_INVAL;
  if (!r.done) return BM_E_STATE;
  r.used = false;
  e.n_live_reqs -= 1;
  return BM_OK;
}

bm_status bm_read_results_many(bm_engine* h, uint64_t first_id, int n, float* hh, float* cc,
                               int32_t* toks, int release) {
  if (h == nullptr || n < 1) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  e.pdl_ok = false;  // other stream work follows: the next launch is fully ordered
  if (e.sticky_cuda) return BM_E_CUDA;
  if (!e.device()) return BM_E_STATE;
  const uint64_t R = e.cfg.max_requests;
  if (static_cast<uint64_t>(n) > R) return BM_E_INVAL;
  for (int i = 0; i < n; ++i) {
    const Request& r = e.reqs[(first_id + i) % R];
    if (!r.used || r.id != first_id + i) return BM_E_INVAL;
    if (!r.done) return BM_E_STATE;
  }
  const size_t LH = e.H() * e.cfg.pool_layers;
  const size_t D = e.cfg.max_decode_len;
  int done = 0;
  while (done < n) {  // contiguous table ranges (the table is a ring)
    const size_t ri = (first_id + done) % R;
    const int len = static_cast<int>(std::min<uint64_t>(n - done, R - ri));
    if (hh) CK(cudaMemcpyAsync(hh + done * LH, e.res_h + ri * LH, len * LH * 4, cudaMemcpyDeviceToHost, e.stream));
    if (cc) CK(cudaMemcpyAsync(cc + done * LH, e.res_c + ri * LH, len * LH * 4, cudaMemcpyDeviceToHost, e.stream));
    if (toks) CK(cudaMemcpyAsync(toks + done * D, e.res_tok + ri * D, len * D * 4, cudaMemcpyDeviceToHost, e.stream));
    done += len;
  }
  CK(cudaStreamSynchronize(e.stream));
  if (toks) {  // as bm_read_result: after an <eos> (N1) the remaining entries are -1
    for (int i = 0; i < n; ++i) {
      const Request& r = e.reqs[(first_id + i) % R];
      if (r.kind != BM_REQ_SEQ2SEQ) continue;
      const int T = r.eos_step >= 0 ? r.eos_step + 1 : r.n_nodes - r.enc_len;
      for (size_t s = T; s < D; ++s) toks[i * D + s] = -1;
    }
  }
  if (release) {
    for (int i = 0; i < n; ++i) {
      Request& r = e.reqs[(first_id + i) % R];
      r.used = false;
      e.n_live_reqs -= 1;
    }
  }
  return BM_OK;
}

bm_status bm_read_log(bm_engine* h, bm_task_record* out, int cap, int* n) {
  if (h == nullptr || n == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  const int k = std::min<int>(cap, static_cast<int>(e.log_tasks.size()));
  if (k > 0) memcpy(out, e.log_tasks.data(), k * sizeof(bm_task_record));
  *n = static_cast<int>(e.log_tasks.size());
  return BM_OK;
}

bm_status bm_read_log_rows(bm_engine* h, bm_row_record* out, int cap, int* n) {
  if (h == nullptr || n == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  const int k = std::min<int>(cap, static_cast<int>(e.log_rows.size()));
  if (k > 0) memcpy(out, e.log_rows.data(), k * sizeof(bm_row_record));
  *n = static_cast<int>(e.log_rows.size());
  return BM_OK;
}

bm_status bm_cell_step(bm_engine* h, int cell_id, const bm_step_row* rows, int b, int async) {
  if (h == nullptr || rows == nullptr || b < 1 || b > 4096) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  if (e.sticky_cuda) return BM_E_CUDA;
  if (!e.device()) return BM_E_STATE;
  if (cell_id < 0 || cell_id >= static_cast<int>(e.cells.size())) return BM_E_INVAL;
  Cell& c = e.cells[cell_id];
  if (c.d.kind == BM_CELL_LSTM_PROJ && b > 512) return BM_E_INVAL;
  for (int i = 0; i < b; ++i) {
    if (rows[i].slot < 0 || rows[i].slot >= e.cfg.max_slots) return BM_E_INVAL;
    if ((rows[i].flags >> 8) >= e.cfg.max_requests) return BM_E_INVAL;
  }
  // tcgen05 path, b <= 512: the rows travel inline with the launch
  const bool inline_rows = e.cfg.precision == BM_PREC_BF16 && b <= kMaxRowsInline;
  const RowDesc* rows_host = inline_rows ? reinterpret_cast<const RowDesc*>(rows) : nullptr;
  // otherwise stage through pinned memory so the copy is truly asynchronous (back-to-back steps)
  if (e.direct_host == nullptr)
    CK(cudaHostAlloc(reinterpret_cast<void**>(&e.direct_host), sizeof(RowDesc) * 4096 * 2, cudaHostAllocDefault));
  RowDesc* rows_dev = nullptr;
  if (!inline_rows) {
    e.pdl_ok = false;
    RowDesc* stage = e.direct_host + (e.direct_flip ^= 1) * 4096;
    if (async) CK(cudaEventSynchronize(e.direct_ev[e.direct_flip]));
    memcpy(stage, rows, sizeof(RowDesc) * b);
    CK(cudaMemcpyAsync(e.direct_rows + e.direct_flip * 4096, stage, sizeof(RowDesc) * b, cudaMemcpyHostToDevice,
                       e.stream));
    CK(cudaEventRecord(e.direct_ev[e.direct_flip], e.stream));
    rows_dev = e.direct_rows + e.direct_flip * 4096;
  }
  // diagnostics: BM_REPEAT=n launches the step n times back to back (steady-state throughput
  // with PDL overlap between consecutive launches; the state advances n steps)
  static const int repeat = getenv("BM_REPEAT") ? atoi(getenv("BM_REPEAT")) : 1;
  for (int rep = 1; rep < repeat; ++rep) {
    bm_status s0 = launch_cell(e, c, rows_dev, rows_host, b, nullptr, nullptr);
    if (s0 != BM_OK) return s0;
  }
  // diagnostics: BM_PHASE_DUMP=<file> records per-CTA phase timestamps of every direct step
  static const char* dump = getenv("BM_PHASE_DUMP");
  if (dump != nullptr && e.phase_dev == nullptr) CK(cudaMalloc(&e.phase_dev, 8 * 64 * 4096));
  if (e.phase_dev) {
    CK(cudaMemsetAsync(e.phase_dev, 0, 8 * 64 * 4096, e.stream));
    e.pdl_ok = false;
  }
  bm_status s = launch_cell(e, c, rows_dev, rows_host, b, nullptr, nullptr);
  if (s != BM_OK) return s;
  if (!async || e.phase_dev) CK(cudaStreamSynchronize(e.stream));
  if (e.phase_dev) {
    std::vector<unsigned long long> h(64 * 4096);
    CK(cudaMemcpy(h.data(), e.phase_dev, h.size() * 8, cudaMemcpyDeviceToHost));
    FILE* f = fopen(dump, "a");
    if (f) {
      fprintf(f, "step b=%d cell=%d\n", b, cell_id);
      for (int i = 0; i < 4096; ++i)
        if (h[i * 64]) {
          fprintf(f, "%d", i);
          for (int k = 0; k < 64; ++k) fprintf(f, " %llu", h[i * 64 + k]);
          fprintf(f, "\n");
        }
      fclose(f);
    }
  }
  return BM_OK;
}

static bm_status pool_io(Engine& e, int layer, int parity, const int32_t* slots, int n, float* h,
                         float* c, int write) {
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  e.pdl_ok = false;
  if (!e.device()) return BM_E_STATE;
  if (layer < 0 || layer >= e.cfg.pool_layers || parity < 0 || parity > 1 || n < 1 || slots == nullptr)
    return BM_E_INVAL;
  for (int i = 0; i < n; ++i)
    if (slots[i] < 0 || slots[i] >= e.cfg.max_slots) return BM_E_INVAL;
  const size_t H = e.H();
  int32_t* ds = nullptr;
  float *dh = nullptr, *dc = nullptr;
  CK(cudaMalloc(&ds, n * 4));
  CK(cudaMalloc(&dh, n * H * 4));
  CK(cudaMalloc(&dc, n * H * 4));
  // every copy is ordered on the engine stream (a pageable cudaMemcpy on the legacy stream
  // may still be in flight when a kernel on the non-blocking engine stream starts)
  CK(cudaMemcpyAsync(ds, slots, n * 4, cudaMemcpyHostToDevice, e.stream));
  if (write) {
    if (h) CK(cudaMemcpyAsync(dh, h, n * H * 4, cudaMemcpyHostToDevice, e.stream));
    if (c) CK(cudaMemcpyAsync(dc, c, n * H * 4, cudaMemcpyHostToDevice, e.stream));
  }
  void* hp = static_cast<char*>(e.h_layer(layer)) + static_cast<size_t>(parity) * e.cfg.max_slots * H * e.elem();
  CK(launch_pool_io(hp, e.c_layer(layer), ds, n, static_cast<int>(H), h ? dh : nullptr,
                    c ? dc : nullptr, write, e.cfg.precision == BM_PREC_BF16, e.stream));
  CK(cudaStreamSynchronize(e.stream));
  if (!write) {
    if (h) CK(cudaMemcpyAsync(h, dh, n * H * 4, cudaMemcpyDeviceToHost, e.stream));
    if (c) CK(cudaMemcpyAsync(c, dc, n * H * 4, cudaMemcpyDeviceToHost, e.stream));
    CK(cudaStreamSynchronize(e.stream));
  }
  cudaFree(ds);
  cudaFree(dh);
  cudaFree(dc);
  return BM_OK;
}

bm_status bm_pool_write(bm_engine* h, int layer, int parity, const int32_t* slots, int n,
                        const float* hh, const float* cc) {
  if (h == nullptr) return BM_E_INVAL;
  return pool_io(*reinterpret_cast<Engine*>(h), layer, parity, slots, n, const_cast<float*>(hh),
                 const_cast<float*>(cc), 1);
}

bm_status bm_pool_read(bm_engine* h, int layer, int parity, const int32_t* slots, int n, float* hh,
                       float* cc) {
  if (h == nullptr) return BM_E_INVAL;
  return pool_io(*reinterpret_cast<Engine*>(h), layer, parity, slots, n, hh, cc, 0);
}

bm_status bm_result_rows(bm_engine* h, const int32_t* res_idx, int n, float* hh, float* cc) {
  if (h == nullptr || res_idx == nullptr || n < 1) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  e.pdl_ok = false;  // other stream work follows: the next launch is fully ordered
  if (!e.device()) return BM_E_STATE;
  const size_t LH = e.H() * e.cfg.pool_layers;
  CK(cudaStreamSynchronize(e.stream));
  for (int i = 0; i < n; ++i) {
    if (res_idx[i] < 0 || res_idx[i] >= e.cfg.max_requests) return BM_E_INVAL;
    if (hh) CK(cudaMemcpyAsync(hh + i * LH, e.res_h + res_idx[i] * LH, LH * 4, cudaMemcpyDeviceToHost, e.stream));
    if (cc) CK(cudaMemcpyAsync(cc + i * LH, e.res_c + res_idx[i] * LH, LH * 4, cudaMemcpyDeviceToHost, e.stream));
  }
  CK(cudaStreamSynchronize(e.stream));
  return BM_OK;
}

bm_status bm_tokens(bm_engine* h, const int32_t* slots, int n, int32_t* inout, int write) {
  if (h == nullptr || slots == nullptr || inout == nullptr || n < 1) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  e.pdl_ok = false;  // other stream work follows: the next launch is fully ordered
  if (!e.device()) return BM_E_STATE;
  CK(cudaStreamSynchronize(e.stream));
  for (int i = 0; i < n; ++i) {
    if (slots[i] < 0 || slots[i] >= e.cfg.max_slots) return BM_E_INVAL;
    if (write) CK(cudaMemcpyAsync(e.tok + slots[i], inout + i, 4, cudaMemcpyHostToDevice, e.stream));
    else CK(cudaMemcpyAsync(inout + i, e.tok + slots[i], 4, cudaMemcpyDeviceToHost, e.stream));
  }
  CK(cudaStreamSynchronize(e.stream));
  return BM_OK;
}

bm_status bm_get_stats(bm_engine* h, bm_stats* out) {
  if (h == nullptr || out == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  *out = e.stats;
  out->kernel_launches = e.stats.kernel_launches - e.launches_base;
  if (e.spans != nullptr) {  // device-side spans accumulated since the last reset
    unsigned long long acc[2 * BM_K_CLASSES];
    CK(cudaStreamSynchronize(e.stream));
    CK(cudaMemcpy(acc, e.spans + 128, sizeof(acc), cudaMemcpyDeviceToHost));
    for (int k = 0; k < BM_K_CLASSES; ++k) {
      out->k_span_ms[k] = (acc[2 * k] - e.span_base[2 * k]) * 1e-6;
      out->k_span_launches[k] = acc[2 * k + 1] - e.span_base[2 * k + 1];
    }
  }
  return BM_OK;
}

bm_status bm_reset_stats(bm_engine* h) {
  if (h == nullptr) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  const uint64_t launches = e.stats.kernel_launches;  // keeps the span slot rotation aligned
  e.stats = bm_stats{};
  e.stats.kernel_launches = launches;
  e.launches_base = launches;
  e.timed_base = e.timed_total;
  if (e.spans != nullptr) {
    CK(cudaStreamSynchronize(e.stream));
    CK(cudaMemcpy(e.span_base, e.spans + 128, sizeof(e.span_base), cudaMemcpyDeviceToHost));
  }
  return BM_OK;
}

bm_status bm_read_launch_log(bm_engine* h, bm_launch_record* out, int cap, int* n) {
  if (h == nullptr || n == nullptr || (cap > 0 && out == nullptr)) return BM_E_INVAL;
  Engine& e = *reinterpret_cast<Engine*>(h);
  std::lock_guard<std::recursive_mutex> lk(e.mu);
  *n = 0;
  if (e.span_log == nullptr) return BM_E_STATE;
  const uint64_t total = e.timed_total - e.timed_base;
  const uint64_t avail = std::min<uint64_t>(total, Engine::kLaunchLog);
  const int k = static_cast<int>(std::min<uint64_t>(avail, static_cast<uint64_t>(std::max(cap, 0))));
  if (k == 0) {
    *n = static_cast<int>(avail);
    return BM_OK;
  }
  std::vector<unsigned long long> spans(Engine::kLaunchLog);
  CK(cudaStreamSynchronize(e.stream));
  CK(cudaMemcpy(spans.data(), e.span_log, spans.size() * 8, cudaMemcpyDeviceToHost));
  const uint64_t first = e.timed_total - avail;
  for (int i = 0; i < k; ++i) {
    const uint64_t li = (first + i) % Engine::kLaunchLog;
    out[i].kclass = e.launch_class[li];
    out[i].b = e.launch_b[li];
    out[i].span_ns = spans[li];
  }
  *n = k;
  return BM_OK;
}

}  // extern "C"
