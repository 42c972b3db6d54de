/*
 * bm.h -- C-ABI of the B200-native cellular-batching engine (BatchMaker, EuroSys'18).
 *
 * One engine drives one GPU. It owns: the loaded cells (packed, device-resident weights),
 * the slot-indexed HBM state pool, the host cell scheduler (Algorithm 1) and the launch /
 * completion path. Everything crossing this boundary is plain C: status codes, plain
 * pointers and sizes. No exceptions, no C++ or torch types.
 *
 * Paper passages (PAPER.md line numbers, /root/reference):
 *   problem statement: users give cell definitions + weights and an unfold rule ... L275 (§4.1)
 *   startup loads each cell and embeds its weights ............................. L319 (§4.2)
 *   requests are unfolded into a cell graph; nodes become ready as inputs do .... L323 (§4.2)
 *   a request returns as soon as its last cell finishes ......................... L331, L267
 *   Schedule(worker) runs when a worker becomes idle ............................. L371 (§4.3)
 *   completion is detected by polling a signal counter in pinned host memory .... L393-L395 (§5)
 *
 * Threading: every call on an engine takes that engine's lock, so calls from several threads
 * are serialised and safe. In particular bm_poll may run on a dedicated polling thread (the
 * paper's poll thread, L395) while another thread submits and schedules; bm_run takes the
 * lock once per round of its event loop, so a concurrent bm_poll interleaves between rounds.
 * Different engines (one per GPU) are independent.
 *
 * Error behaviour: every call returns a bm_status. BM_E_CUDA is sticky: after it every
 * call that touches the device returns BM_E_CUDA again and the engine can only be
 * destroyed. All other errors leave the engine unchanged (the call had no effect).
 */
#ifndef BM_H_
#define BM_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BM_ABI_VERSION 1

typedef struct bm_engine bm_engine; /* opaque; owns all its host and device memory */

typedef enum {
  BM_OK = 0,
  BM_E_INVAL = -1, /* malformed argument: bad sizes, malformed tree, token >= vocab, ...  */
  BM_E_NOMEM = -2, /* host or device allocation failed                                     */
  BM_E_FULL = -3,  /* request table full: back-pressure, retry after bm_poll retires some  */
  BM_E_AGAIN = -4, /* nothing to do now (bm_schedule_step: idle worker, nothing ready)     */
  BM_E_CUDA = -5,  /* CUDA error; sticky                                                   */
  BM_E_STATE = -6, /* call not valid in the current state (e.g. cell loaded after submit)  */
  BM_E_NODEV = -7  /* no usable sm_100 device (the library never falls back to the CPU)    */
} bm_status;

/* Arithmetic of the cell kernels. BF16: bf16 weights/activations, fp32 accumulation in
 * TMEM (tcgen05), fp32 cell state c. FP32: fp32 weights/activations/state on SIMT FFMA
 * (parity path, north_star tolerance 1e-5). */
enum { BM_PREC_BF16 = 0, BM_PREC_FP32 = 1 };

/* Clock the scheduler runs on.
 * BM_CLOCK_WALL:    arrivals are seconds relative to bm_run's start; tasks retire when the
 *                   device signals them.
 * BM_CLOCK_VIRTUAL: arrivals are ticks; every task takes exactly one tick on the worker
 *                   (Figure 5's model, L269). The GPU still executes every task; retire
 *                   order and the log are a pure function of the trace (bit-exact replay).
 * BM_CLOCK_DRY:     as VIRTUAL but no device work at all (no GPU needed): the scheduler,
 *                   request processor and slot pool alone, for host-side tests. */
enum { BM_CLOCK_WALL = 0, BM_CLOCK_VIRTUAL = 1, BM_CLOCK_DRY = 2 };

typedef struct {
  int device;        /* CUDA ordinal the engine binds to                                  */
  int precision;     /* BM_PREC_*                                                         */
  int clock;         /* BM_CLOCK_*                                                        */
  int hidden;        /* h of the state pool; every loaded cell must use this h            */
  int pool_layers;   /* layers per slot (max over loaded LSTM stacks; 1 for trees)        */
  int max_slots;     /* slots in the HBM state pool                                       */
  int max_requests;  /* request table entries (in-flight + completed-but-unreleased)      */
  int max_tasks_to_submit;   /* Algorithm 1 MaxTasksToSubmit, default 5 (L379)            */
  int min_followon_batch;    /* Algorithm 1 Bsizes.Min() (reading S14), default 1         */
  int schedule_when_outstanding_leq; /* Schedule when <= k tasks outstanding; 0 = idle (S19) */
  int max_decode_len;        /* decoder tokens kept per request (result buffer)           */
  int keep_results;          /* 1: results stay readable until bm_release; 0: auto-free  */
  int record_logits;         /* debug: keep every decode step's logits (parity tests)     */
  int time_kernels;          /* 1: device-time EVERY kernel launch (per-kernel roofline,  */
                             /* bm_stats.k_*, bm_read_launch_log)                          */
  int record_log;            /* 1: keep the task log for bm_read_log (default 1)          */
  int persistent;            /* 1: bm_run serves an engine whose only cell is a 1-layer   */
                             /* LSTM with one persistent, weight-stationary kernel (its   */
                             /* weight slice stays in shared memory; tasks arrive through */
                             /* a device ring; a grid barrier separates tasks). Ignored   */
                             /* (regular launches) when the engine is not eligible.       */
  int policy;                /* BM_POLICY_*: cellular batching (Algorithm 1, default) or  */
                             /* the padding + bucketing graph-batching baseline (§7.1,    */
                             /* L427-L437; chain requests only)                            */
  int bucket_width;          /* graph batching: bucket i holds lengths (i*w, (i+1)*w] and */
                             /* its graph is unrolled to (i+1)*w steps (L427, L631); 10    */
  int workers;               /* Algorithm 1 workers of this engine (§4, §8f N2), one */
                             /* stream each on the engine's device; Schedule(worker) runs */
                             /* for each idle worker, FormBatchedTask skips subgraphs     */
                             /* pinned to another worker (Alg. 1 line 27, L381). 1 =      */
                             /* request sharding's one worker per GPU (default). >1 needs */
                             /* policy CELLULAR and persistent 0; the bf16 LSTM launches  */
                             /* then use a <= 113 KB plan so two workers' CTAs share SMs. */
  int devices;               /* device contexts the workers spread over (§8f N2, the paper's */
                             /* multi-GPU design, L317, L337): worker w runs on context w %  */
                             /* devices, context c on CUDA device (device + c) % count. A    */
                             /* context holds its own weight replica and state pool; when a  */
                             /* subgraph is scheduled on a worker of another context (it is  */
                             /* unpinned: nothing of it in flight, L381), its state rows move */
                             /* with it by peer copies ("if the execution of successive cells */
                             /* switch from one GPU to another, one must copy data", L337),  */
                             /* counted in bm_stats.migrations. Results land on context 0.  */
                             /* 1 = one context (default); > 1 needs workers >= devices.    */
  double roof_hbm_gbs;       /* time_kernels: the roofline denominators (bench.py passes     */
  double roof_tc_tflops;     /* MEASURED_PEAKS.json); 0 = bm_stats.k_roof_* stay 0          */
} bm_config;

enum {
  BM_POLICY_CELLULAR = 0,    /* Algorithm 1 (L345-L369): requests join / leave between cells */
  BM_POLICY_GRAPH = 1        /* padding + bucketing, round robin over buckets, a batch runs */
                             /* its whole padded graph and returns all outputs at its end  */
};

/* Fill *cfg with defaults: device 0, BF16, WALL, hidden 1024, 1 layer, 65536 slots,
 * 65536 requests, MaxTasksToSubmit 5, Min 1, k 0, max_decode_len 512, keep_results 0,
 * record_log 1, persistent 0, policy BM_POLICY_CELLULAR, bucket_width 10, workers 1,
 * devices 1. */
void bm_config_default(bm_config* cfg);

/* ---------------------------------------------------------------- cells (bm_load_cell) */
enum {
  BM_CELL_LSTM = 0,        /* L-layer LSTM stack, one node = one timestep (M1-M3)       */
  BM_CELL_LSTM_PROJ = 1,   /* decoder: LSTM stack + output projection + argmax (M4)     */
  BM_CELL_TREE_LEAF = 2,   /* TreeLSTM leaf (M5)                                        */
  BM_CELL_TREE_INTERNAL = 3 /* TreeLSTM binary internal node (M6)                        */
};

typedef struct {
  int kind;       /* BM_CELL_*                                                          */
  int hidden;     /* h (must equal bm_config.hidden)                                    */
  int layers;     /* LSTM stacks: 1..pool_layers; trees: 1                              */
  int vocab;      /* rows of the embedding E (and of W_out for BM_CELL_LSTM_PROJ)       */
  int max_batch;  /* bmax of this cell type = Bsizes.Max() (L323, L345), <= 512         */
  int priority;   /* larger = scheduled first among equals (L339, Alg. 1 line 10)       */
} bm_cell_desc;

/* Weights in the paper/oracle layout, row-major fp32 (startup loads each cell and "embeds"
 * its weights, L319). Each pointer may be a HOST pointer (copied up) or a DEVICE pointer on
 * the engine's device (adopted in place: the packing kernels read it directly, so weights
 * broadcast once with NCCL land without a host round trip); a device pointer
 * of another device is BM_E_INVAL. The library keeps its own packed copy; the caller keeps
 * ownership and may free the arrays after the call. In BF16 precision they are rounded to
 * bf16 (round-to-nearest-even) and packed on the device by the library.
 *   BM_CELL_LSTM / _PROJ: W[l] = [4h, 2h] acting on the column [x; h], gate row blocks
 *                         (i, f, g, o); b[l] = [4h]; E = [vocab, h];
 *                         _PROJ adds W_out = [vocab, h], b_out = [vocab].
 *   BM_CELL_TREE_LEAF:     W[0] = W_leaf [3h, h], gate blocks (i, o, u); b[0] = [3h]; E.
 *   BM_CELL_TREE_INTERNAL: W[0] = U [5h, 2h] acting on [h_L; h_R], gate blocks
 *                          (i, f_L, f_R, o, u); b[0] = [5h]; E unused (NULL).       */
typedef struct {
  const float* const* W;
  const float* const* b;
  const float* E;
  const float* W_out;
  const float* b_out;
} bm_weights;

/* Load one cell type; returns its id (0, 1, ...) in *cell_id. Must precede bm_submit.
 * Errors: BM_E_INVAL (shape mismatch with the config), BM_E_NOMEM, BM_E_CUDA, BM_E_STATE. */
bm_status bm_load_cell(bm_engine* e, const bm_cell_desc* desc, const bm_weights* w,
                       int* cell_id);

/* ---------------------------------------------------------------- requests (bm_submit) */
enum { BM_REQ_CHAIN = 0, BM_REQ_SEQ2SEQ = 1, BM_REQ_TREE = 2 };

typedef struct {
  int kind;            /* BM_REQ_*                                                        */
  int cell0, cell1;    /* CHAIN: cell0; SEQ2SEQ: encoder, decoder; TREE: leaf, internal   */
  int n;               /* CHAIN/SEQ2SEQ: tokens (source length, >= 1); TREE: nodes        */
  const int32_t* tokens;   /* [n]; TREE: word id per node (read at leaves only)           */
  int decode_len;      /* SEQ2SEQ: decoder steps T >= 1 (exactly T, L715)                 */
  const int32_t* left;     /* TREE: [n] left child or -1 (leaf); post-order, root = n-1   */
  const int32_t* right;    /* TREE: [n] right child or -1                                 */
  double arrival;      /* WALL: seconds after bm_run start; VIRTUAL/DRY: tick             */
  uint64_t user_tag;   /* returned in bm_completion                                       */
  /* SEQ2SEQ <eos>-terminated decoding (L715: "Decoding terminates when either
   * the <eos> symbol is generated or when the maximum decoding length is reached"). eos_stop
   * = 0 (zero-initialised default): decode exactly decode_len steps (the paper's protocol).
   * eos_stop = 1: decode_len is the maximum length (<= 4095); the device marks the request
   * finished when its argmax equals eos_id (0 <= eos_id < vocab); decoder steps the scheduler
   * had already submitted (look-ahead, L379) are masked on the device and nothing further is
   * scheduled. The scheduler learns of the <eos> at the retire of the task that emitted it.
   * dry_eos_step: BM_CLOCK_DRY only (no device, scheduler tests): the decode step whose token
   * the scheduler is told was <eos> (-1 = never).                                            */
  int eos_stop;
  int32_t eos_id;
  int dry_eos_step;
} bm_request;

/* Admit a request (unfold, A1). All arrays are copied. The request becomes visible to the
 * scheduler once the clock reaches `arrival` ("When a new request arrives, the request
 * processor runs the user-code to unfold the recursion", L323). *req_id = admission index
 * (0, 1, 2, ...). Requests not yet admitted form an arrival stream: `arrival` must be >= the
 * arrival of every earlier-submitted request that is still pending (BM_E_INVAL otherwise).
 * Errors: BM_E_INVAL (bad cell kinds, token out of range, tree not binary/post-order,
 * arrival earlier than a pending request's),
 * BM_E_FULL (request table full; retry after retiring), BM_E_STATE. */
bm_status bm_submit(bm_engine* e, const bm_request* r, uint64_t* req_id);

/* Admit n requests in one call (same semantics as n bm_submit calls, stops at the first
 * failure). *first_id = id of reqs[0]; ids are consecutive. *n_done = requests accepted. */
bm_status bm_submit_many(bm_engine* e, const bm_request* reqs, int n, uint64_t* first_id,
                         int* n_done);

/* One scheduler round at the current clock: retire what the device finished, admit due
 * arrivals, and if the worker is idle (<= k outstanding tasks) run Schedule(worker)
 * (Algorithm 1), launching every formed task. *n_tasks = tasks launched (may be 0).
 * VIRTUAL/DRY clocks: the clock then advances to the next event tick.
 * Returns BM_E_AGAIN when nothing is outstanding, nothing is ready and nothing is
 * pending (everything submitted so far has completed). */
bm_status bm_schedule_step(bm_engine* e, int* n_tasks);

typedef struct {
  uint64_t req_id;
  uint64_t user_tag;
  double t_arrival;      /* seconds (WALL) or ticks                                       */
  double t_first;        /* first node scheduled                                          */
  double t_done;         /* retire of the last node                                       */
} bm_completion;

/* Non-blocking: copies up to cap completions (in completion order) not yet returned. */
bm_status bm_poll(bm_engine* e, bm_completion* out, int cap, int* n);

/* Drive the event loop until every submitted request has completed (the open-loop driver
 * used by bench.py: arrivals released at their time, Schedule on idle, polling retire).
 * *n_completed = requests completed by this call. */
bm_status bm_run(bm_engine* e, int* n_completed);

typedef struct {
  float* h;          /* [layers][hidden] final hidden state (fp32), or NULL              */
  float* c;          /* [layers][hidden] final cell state, or NULL                       */
  int32_t* tokens;   /* SEQ2SEQ: [decode_len] emitted tokens, or NULL; with eos_stop the
                        entries after the <eos> step are -1                                 */
  float* logits;     /* SEQ2SEQ with record_logits: [decode_len][vocab], or NULL          */
} bm_result;

/* Synchronous copy of a completed request's results into caller-owned buffers.
 * Errors: BM_E_INVAL (unknown id), BM_E_STATE (not completed / already released). */
bm_status bm_read_result(bm_engine* e, uint64_t req_id, bm_result* dst);
bm_status bm_release(bm_engine* e, uint64_t req_id);

/* Bulk result read for the consecutive ids [first_id, first_id + n), all completed and kept:
 * one device->host copy per contiguous table range. h, c: [n][pool_layers][hidden] fp32 or
 * NULL; tokens: [n][max_decode_len] or NULL (entries past a request's last emitted token are
 * -1). Then releases them if release != 0. */
bm_status bm_read_results_many(bm_engine* e, uint64_t first_id, int n, float* h, float* c,
                               int32_t* tokens, int release);

/* Task log (replay parity, P9): one record per launched task, rows flattened. */
typedef struct {
  int task;        /* launch index                                                        */
  int cell;        /* cell type id                                                        */
  double tick;     /* submit time (tick or seconds)                                       */
  int first_row;   /* index into the rows array returned by bm_read_log_rows             */
  int n_rows;
  int worker;      /* Algorithm 1 worker that ran the task (bm_config.workers)            */
} bm_task_record;

typedef struct {
  uint64_t req_id;
  int node;        /* request-local node index                                            */
  int slot;        /* output slot of the row                                              */
} bm_row_record;

bm_status bm_read_log(bm_engine* e, bm_task_record* out, int cap, int* n);
bm_status bm_read_log_rows(bm_engine* e, bm_row_record* out, int cap, int* n);

/* ---------------------------------------------------------------- direct cell access
 * Kernel-level entry points used by the parity tests and the roofline measurement: run ONE
 * batched cell step of a loaded cell over an arbitrary (non-contiguous) set of pool slots,
 * bypassing the scheduler. rows[b] as bm_step_row; device work is synchronous on return
 * unless `async` is nonzero. */
typedef struct {
  int32_t a;       /* LSTM/leaf: token id (-1: use the device feed token tok[slot]);
                      internal: left child slot                                           */
  int32_t b;       /* internal: right child slot; decoder: decode step index              */
  int32_t slot;    /* output slot (LSTM: also the state read)                             */
  int32_t flags;   /* BM_ROW_* | (result_index << 8)                                      */
} bm_step_row;

enum { BM_ROW_FIRST = 1,  /* h_prev = c_prev = 0 (first node of a request)                 */
       BM_ROW_LAST = 2,   /* write fp32 h, c of this row to result row (flags >> 8)        */
       BM_ROW_PARITY = 4, /* LSTM: read h[parity], write h[1 - parity]                     */
       BM_ROW_EOS = 8     /* decoder row of an eos_stop request: b = step | (eos_id + 1) << 12;
                             the row is a no-op once the slot's request emitted <eos>      */ };

bm_status bm_cell_step(bm_engine* e, int cell_id, const bm_step_row* rows, int b, int async);

/* Pool access (tests): copy fp32 state of `n` slots in/out. layer < pool_layers,
 * parity in {0,1} selects the h buffer. h/c are [n][hidden] fp32 host arrays. */
bm_status bm_pool_write(bm_engine* e, int layer, int parity, const int32_t* slots, int n,
                        const float* h, const float* c);
bm_status bm_pool_read(bm_engine* e, int layer, int parity, const int32_t* slots, int n,
                       float* h, float* c);
/* Result rows written by BM_ROW_LAST rows. h/c: [n][layers][hidden]. */
bm_status bm_result_rows(bm_engine* e, const int32_t* res_idx, int n, float* h, float* c);
/* Device feed tokens tok[slot] (decoder) in/out. */
bm_status bm_tokens(bm_engine* e, const int32_t* slots, int n, int32_t* inout, int write);

/* ---------------------------------------------------------------- measurement
 * Per-kernel roofline accounting (time_kernels = 1). EVERY launch is timed on the device: its
 * span runs from the first CTA past its dependency wait (the point where the launch's
 * dependent work may begin; under PDL its setup overlaps the previous launch) to the last CTA
 * done (%globaltimer), accumulated per kernel class by the launch's last CTA. The host adds
 * the same launch's ALGORITHMIC bytes and flops (weights streamed once,
 * gathered operand rows, state read/written; padding not counted) to the same class, so
 * bytes, flops and time always cover one population. k_roof_* sum, per launch, the time the
 * launch would take at the roof: bytes / roof_hbm_gbs, flops / roof_tc_tflops, and the larger
 * of the two (the launch's binding roof: HBM below the ridge, tensor above). */
enum {
  BM_K_LSTM_PAIR = 0,   /* cell_pair_kernel: LSTM layer, tcgen05 cta_group::2 (129-512 rows) */
  BM_K_LSTM = 1,        /* cell_step_sm100_kernel<EPI_LSTM>                                  */
  BM_K_LEAF = 2,        /* cell_step_sm100_kernel<EPI_LEAF>                                  */
  BM_K_INTERNAL = 3,    /* cell_step_sm100_kernel<EPI_INTERNAL>                              */
  BM_K_PROJ = 4,        /* decoder projection + argmax                                       */
  BM_K_SIMT = 5,        /* fp32 SIMT parity path (all cell kinds)                            */
  BM_K_PERSISTENT = 6,  /* persistent weight-stationary LSTM: one "launch" = one task        */
  BM_K_CLASSES = 8
};

typedef struct {
  uint64_t tasks;            /* tasks launched                                           */
  uint64_t rows;             /* rows (cell nodes) executed                               */
  uint64_t kernel_launches;  /* our kernels launched                                     */
  double sched_ns;           /* host time spent in Schedule/Batch                        */
  uint64_t schedule_calls;
  double launch_ns;          /* host time spent staging descriptors and issuing launches  */
  double retire_ns;          /* host time spent retiring finished tasks (Retire, A4)      */
  uint64_t k_launches[BM_K_CLASSES];      /* launches issued, per class                  */
  uint64_t k_span_launches[BM_K_CLASSES]; /* launches whose device span landed (equal to */
                                          /* k_launches once the device is idle)          */
  double k_span_ms[BM_K_CLASSES];         /* sum of device spans                         */
  double k_rows[BM_K_CLASSES];            /* sum of rows (b) over the launches           */
  double k_bytes[BM_K_CLASSES];           /* sum of algorithmic bytes                    */
  double k_flops[BM_K_CLASSES];           /* sum of algorithmic flops                    */
  double k_roof_hbm_ms[BM_K_CLASSES];     /* sum of bytes / roof_hbm_gbs                 */
  double k_roof_tc_ms[BM_K_CLASSES];      /* sum of flops / roof_tc_tflops               */
  double k_roof_ms[BM_K_CLASSES];         /* sum of max(the two) per launch              */
  uint64_t migrations;       /* state rows moved between device contexts (bm_config.devices) */
  double migration_bytes;    /* bytes those peer copies moved                               */
} bm_stats;

bm_status bm_get_stats(bm_engine* e, bm_stats* out);
bm_status bm_reset_stats(bm_engine* e);

/* Launch log (time_kernels = 1): the last <= 65536 launches since bm_reset_stats, oldest
 * first: kernel class, rows, device span in ns (0 if not landed). Synchronises the stream. */
typedef struct {
  int kclass;
  int b;
  uint64_t span_ns;
} bm_launch_record;
bm_status bm_read_launch_log(bm_engine* e, bm_launch_record* out, int cap, int* n);

/* Device stream the engine launches on (cudaStream_t as void*), so callers can bracket
 * runs with CUDA events on that stream. */
void* bm_stream(bm_engine* e);

/* ---------------------------------------------------------------- lifecycle */
bm_status bm_create(const bm_config* cfg, bm_engine** out);
void bm_destroy(bm_engine* e);
const char* bm_strerror(bm_status s);
int bm_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BM_H_ */
