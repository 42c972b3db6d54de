// engine.h -- internal structures of the host runtime behind include/bm.h.
//
//   Engine
//    ├─ cells[]        loaded cell types: packed device weights + TMA maps + scheduler queue
//    ├─ reqs[]         request table (ring of max_requests entries): cell graph + subgraphs
//    ├─ SlotPool       lowest-free-index allocator over the HBM state pool (A4)
//    ├─ Scheduler      Algorithm 1 (Schedule / Batch / FormBatchedTask)
//    ├─ in-flight FIFO tasks launched, not yet retired (the paper's in-progress queue, L331)
//    └─ device         pool h/c, feed tokens, result rows, row-descriptor ring, signal counter
#pragma once
#include <stdint.h>

#include <algorithm>
#include <chrono>
#include <deque>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/bm.h"
#include "kernels.h"

namespace bm {

struct Engine;

// ---------------------------------------------------------------- cell graph (A1, D1-D3)
// Ready nodes of a subgraph, ascending (height, post-order index) [S18]. Chain / Seq2Seq
// subgraphs hold at most one ready node, so small lists live inline (no heap, same cache line).
struct ReadyList {
  int n = 0;
  int inl[2] = {0, 0};
  std::vector<int> big;  // used once n would exceed the inline capacity (tree internal)
  int size() const { return n; }
  int operator[](int i) const { return big.empty() ? inl[i] : big[i]; }
  void clear() {
    n = 0;
    big.clear();
  }
  void assign1(int v) {
    clear();
    inl[0] = v;
    n = 1;
  }
  void insert_at(int pos, int v) {
    if (big.empty() && n < 2) {
      for (int i = n; i > pos; --i) inl[i] = inl[i - 1];
      inl[pos] = v;
      ++n;
      return;
    }
    if (big.empty()) big.assign(inl, inl + n);
    big.insert(big.begin() + pos, v);
    ++n;
  }
  void erase_value(int v) {
    if (big.empty()) {
      int i = 0;
      while (i < n && inl[i] != v) ++i;
      for (; i + 1 < n; ++i) inl[i] = inl[i + 1];
      --n;
      return;
    }
    big.erase(std::find(big.begin(), big.end(), v));
    --n;
    if (n == 0) big.clear();
  }
  bool contains(int v) const {
    for (int i = 0; i < n; ++i)
      if ((*this)[i] == v) return true;
    return false;
  }
};

struct Subgraph {
  int req = -1;            // request table index
  int sid = 0;             // subgraph id within the request
  int ct = 0;              // cell type
  int n_nodes = 0;
  int n_submitted = 0;
  int n_completed = 0;
  int pinned = -1;         // worker id or -1 (Alg. 1 line 21, L381)
  int inflight = 0;        // tasks in flight holding nodes of this subgraph
  // intrusive FIFO links of the cell type's subgraph queue (D3)
  int q_prev_req = -1, q_prev_sid = -1, q_next_req = -1, q_next_sid = -1;
  bool queued = false;
  ReadyList ready;
};

// Hot fields first: the scheduler touches a request several times per scheduled node.
struct Request {
  int kind = 0;
  int cell0 = 0, cell1 = 0;
  int n_nodes = 0;          // chain: L; seq2seq: S + T; tree: n
  int enc_len = 0;          // seq2seq: S
  int n_completed = 0;
  int slot = -1;            // chain / seq2seq
  int leaves_left = 0;
  int internal_sid = -1;
  // <eos>-terminated decoding (§8f N1)
  bool eos_stop = false;
  int eos_id = -1;
  int eos_step = -1;        // decode step of the <eos>, once the scheduler has learned it
  int dry_eos_step = -1;    // BM_CLOCK_DRY: the step reported as <eos>
  int decode_max = 0;       // decode_len as submitted (maximum length under eos_stop)
  bool used = false;
  bool done = false;
  bool started = false;     // slots taken
  uint64_t id = 0;          // admission index
  uint64_t tag = 0;
  double t_arrival = 0, t_first = -1, t_done = -1;
  Subgraph sg2[2];          // chain: [0]; seq2seq: encoder [0], decoder [1]
  std::vector<int32_t> tokens;      // chain/seq2seq: source tokens; tree: per node
  // trees only
  std::vector<Subgraph> sgv;        // leaf subgraphs then the internal subgraph
  std::vector<int32_t> left, right, parent, height, node_slot;
  std::vector<uint8_t> submitted;
  std::vector<int> node_sid;        // subgraph of each node
  Subgraph& sg(int sid) { return kind == BM_REQ_TREE ? sgv[sid] : sg2[sid]; }
  const Subgraph& sg(int sid) const { return kind == BM_REQ_TREE ? sgv[sid] : sg2[sid]; }
  int sid_of(int node) const {
    return kind == BM_REQ_TREE ? node_sid[node] : (kind == BM_REQ_SEQ2SEQ && node >= enc_len ? 1 : 0);
  }
};

struct Cell {
  bm_cell_desc d{};
  int epi = 0, G = 0, U = 0, S = 1, kslice = 0, K0 = 0, K1 = 0;
  // device weights (per layer for LSTM stacks)
  std::vector<void*> W;
  std::vector<float*> bias;
  void* E = nullptr;
  void* W_out = nullptr;
  float* b_out = nullptr;
  // scheduler state of this cell type
  int q_head_req = -1, q_head_sid = -1, q_tail_req = -1, q_tail_sid = -1;
  int64_t ready_nodes = 0;   // NumReadyNodes (S16)
  int running_tasks = 0;     // NumRunningTasks (S17)
};

// Device context (bm_config.devices, §8f N2): the state pool, descriptor ring and the weight
// replica of every cell on one CUDA device. The Engine's own fields (h_pool, c_pool, tok, dead,
// ring_dev, ..., Cell::W/bias/E/W_out/b_out) are the ACTIVE context's; select_worker() swaps
// them with the parked copies here when the next worker lives on another context.
struct CellWeights {
  std::vector<void*> W;
  std::vector<float*> bias;
  void* E = nullptr;
  void* W_out = nullptr;
  float* b_out = nullptr;
};
struct DevCtx {
  int cuda_dev = 0;
  void* h_pool = nullptr;
  float* c_pool = nullptr;
  int* tok = nullptr;
  int* dead = nullptr;
  RowDesc* ring_dev = nullptr;
  RowDesc* ring_host = nullptr;
  int ring_head = 0;
  unsigned int* rows_flag_dev = nullptr;
  unsigned int* rows_seq_host = nullptr;
  unsigned int rows_seq = 0;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t copy_ev = nullptr;
  std::vector<CellWeights> cells;
};

struct TaskRow {
  int req;     // request table index
  int node;
  int slot;
};

struct Task {
  uint64_t seq = 0;          // launch index
  int ct = 0;
  double tick = 0;           // submit time
  double finish = 0;         // VIRTUAL: retire tick
  int ring_off = 0;          // first row in the descriptor ring
  int b = 0;
  std::vector<TaskRow> rows;
  std::vector<RowDesc> desc; // device row descriptors, built at submission (A3)
  std::vector<int> batch_reqs;      // graph batching: the batch's requests (on its last task)
  int worker = 0;                   // Algorithm 1 worker (bm_config.workers)
};

// Launch state of one Algorithm-1 worker (§4, §8f N2): its stream, in-progress queue,
// completion counter, launch chain and per-launch device scratch. The Engine's own copies of
// these fields (stream, inflight, launched, ...) are the ACTIVE worker's; select_worker()
// swaps them with the parked copies, so the launch / retire code serves any worker.
struct WorkerState {
  cudaStream_t stream = nullptr;
  std::deque<Task> inflight;
  uint64_t launched = 0;
  double last_finish = 0;
  unsigned long long* signal_host = nullptr;
  unsigned long long* signal_dev = nullptr;
  unsigned int* dep_flag = nullptr;
  unsigned int dep_seq = 0;
  bool pdl_ok = false;
  unsigned int* sig_ctas = nullptr;
  unsigned int* done_ctas = nullptr;
  unsigned long long* amax = nullptr;
  float* scratch = nullptr;
};


struct Engine {
  std::recursive_mutex mu;          // every C-ABI call on the engine holds it (include/bm.h)
  bm_config cfg{};
  bool sticky_cuda = false;
  bool submitted_any = false;
  std::vector<Cell> cells;
  std::vector<Request> reqs;        // ring of max_requests
  int n_live_reqs = 0;
  uint64_t next_req_id = 0;
  std::deque<int> pending;          // request table indices not yet admitted (FIFO, S21)
  std::vector<std::deque<int>> buckets;  // graph batching: admitted requests per bucket [G1]
  int last_bucket = -1;                  // graph batching: round-robin position
  std::vector<int> free_slots_heap; // min-heap of free slots (A4)
  std::deque<Task> inflight;        // in-progress queue (L331, L395)
  uint64_t launched = 0;            // tasks launched so far (== signal target)
  double now = 0;                   // clock: ticks (VIRTUAL/DRY) or seconds since bm_run
  double last_finish = 0;
  std::chrono::steady_clock::time_point t0;
  bool wall_started = false;
  std::vector<bm_completion> completions;   // not yet returned by bm_poll
  uint64_t completed_total = 0;             // requests completed since creation
  std::vector<bm_task_record> log_tasks;
  std::vector<bm_row_record> log_rows;
  bm_stats stats{};

  // ---- device
  cudaStream_t stream = nullptr;
  void* h_pool = nullptr;          // [layers][2][slots][H]
  float* c_pool = nullptr;         // [layers][slots][H]
  int* tok = nullptr;              // [slots]
  int* dead = nullptr;             // [slots] device: request emitted <eos> (N1)
  int* eos_host = nullptr;         // [max_requests] pinned, mapped: <eos> step + 1 (N1)
  int* eos_dev = nullptr;          // device pointer of eos_host
  float* res_h = nullptr;          // [max_requests][layers][H]
  float* res_c = nullptr;
  int32_t* res_tok = nullptr;      // [max_requests][max_decode]
  float* logits = nullptr;         // [max_requests][max_decode][V] (record_logits)
  int logits_vocab = 0;
  unsigned long long* amax = nullptr;
  float* scratch = nullptr;          // split-K partial exchange of cell_pair2_kernel (L2)
  unsigned int* done_ctas = nullptr;
  unsigned int* sig_ctas = nullptr;  // CTA counter of the fused completion signal / chain flag
  unsigned int* dep_flag = nullptr;  // launch chain flag (device): last completed sm100 launch
  unsigned int dep_seq = 0;          // host: sequence number of the last sm100 launch issued
  bool pdl_ok = false;               // the stream's last op was an sm100 launch (PDL is safe)
  // ring rows of the tcgen05 path: published by a copy + a flag write on copy_stream
  unsigned int* rows_flag_dev = nullptr;   // device: last published rows sequence number
  unsigned int* rows_seq_host = nullptr;   // pinned ring of sequence values (flag-copy fallback)
  unsigned int rows_seq = 0;               // host: last sequence number issued
  unsigned int launch_rows_seq = 0;        // 0: the launch's rows need no flag wait
  void* write_value32 = nullptr;           // cuStreamWriteValue32 (driver entry point) or null
  RowDesc* ring_dev = nullptr;
  RowDesc* ring_host = nullptr;    // pinned staging
  int ring_rows = 0;
  int ring_head = 0;               // next free row
  int ring_used = 0;               // rows held by in-flight tasks
  unsigned long long* signal_host = nullptr;   // pinned, mapped
  unsigned long long* signal_dev = nullptr;
  RowDesc* direct_rows = nullptr;  // bm_cell_step rows (device)
  unsigned long long* phase_dev = nullptr;  // BM_PHASE_DUMP diagnostics
  RowDesc* direct_host = nullptr;  // pinned staging of bm_cell_step rows (double buffered)
  cudaEvent_t direct_ev[2] = {nullptr, nullptr};
  int direct_flip = 0;
  // persistent weight-stationary LSTM (bm_config.persistent)
  bool persistent_active = false;
  cudaStream_t copy_stream = nullptr;  // descriptor-ring copies (off the kernel stream)
  cudaEvent_t copy_ev = nullptr;
  TaskHdr* hdr_dev = nullptr;
  TaskHdr* hdr_host = nullptr;         // pinned staging
  int hdr_ring = 256;
  unsigned int* gbar = nullptr;
  int* perr = nullptr;
  uint64_t run_base = 0;               // launch index of the run's first task
  // per-kernel timing (time_kernels): device [64 span slots x {start, ctas}] then
  // [BM_K_CLASSES x {ns, launches}] accumulators, and a per-launch span log (kLaunchLog)
  static constexpr int kLaunchLog = 1 << 16;
  unsigned long long* spans = nullptr;
  unsigned long long span_base[2 * BM_K_CLASSES] = {};
  unsigned long long* span_log = nullptr;     // device [kLaunchLog] span ns of launch i
  std::vector<int> launch_class, launch_b;    // host [kLaunchLog] class / rows of launch i
  uint64_t timed_total = 0;                   // launches given a span slot so far
  uint64_t timed_base = 0;                    // timed_total at the last bm_reset_stats
  uint64_t poll_spins = 0;                    // non-blocking completion polls (error checks)
  uint64_t launches_base = 0;
  // diagnostics (BM_TIMELINE=<file>): per-launch device times + host issue times, per-task
  // host retire times; written at bm_destroy
  static constexpr uint64_t kTimeline = 8192;
  unsigned long long* tl_dev = nullptr;
  std::vector<long long> tl_host, tl_retire;
  std::vector<int> tl_b;
  uint64_t tl_n = 0;

  // workers (§8f N2): parked launch state of the inactive workers; `cur` is active
  std::vector<WorkerState> parked;
  int cur = 0;
  // device contexts (bm_config.devices): parked state of the inactive contexts, the context
  // of each worker, and the context holding each slot's latest state (-1: none yet)
  std::vector<DevCtx> ctxs;
  int cur_ctx = 0;
  std::vector<int> worker_ctx;
  std::vector<int8_t> slot_ctx;
  uint64_t tasks_total = 0;         // tasks over all workers (task log index)

  bool device() const { return cfg.clock != BM_CLOCK_DRY; }
  std::deque<Task>& inflight_of(int w) { return w == cur ? inflight : parked[w].inflight; }
  size_t elem() const { return cfg.precision == BM_PREC_BF16 ? 2 : 4; }
  size_t H() const { return static_cast<size_t>(cfg.hidden); }
  void* h_layer(int l) const {
    return static_cast<char*>(h_pool) + static_cast<size_t>(l) * 2 * cfg.max_slots * H() * elem();
  }
  float* c_layer(int l) const { return c_pool + static_cast<size_t>(l) * cfg.max_slots * H(); }
};

// scheduler.cpp
bm_status admit_request(Engine& e, int ri);
int schedule(Engine& e, int worker, std::vector<Task>& out);  // Schedule(worker): tasks formed
void retire_task(Engine& e, Task& t);
bool has_ready(const Engine& e);
void slot_release(Engine& e, int s);

// runtime.cpp
void select_worker(Engine& e, int w);
bm_status launch_tasks(Engine& e, std::vector<Task>& tasks);
double wall_now(const Engine& e);

}  // namespace bm
