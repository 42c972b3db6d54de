// Internal interface between the host runtime (engine.cpp) and the sm_100a kernels.
// Not part of the public C-ABI (include/bm.h).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace bm {

// One row of a batched cell task (== bm_step_row in include/bm.h).
struct RowDesc {
  int32_t a;      // LSTM/leaf: token id, or -1 = device feed token tok[slot]; internal: left slot
  int32_t b;      // internal: right slot; decoder projection: decode step index
  int32_t slot;   // output slot (LSTM: also the state read)
  int32_t flags;  // ROW_* | result_index << 8
};
enum { ROW_FIRST = 1, ROW_LAST = 2, ROW_PARITY = 4, ROW_EOS = 8 };
// ROW_EOS rows (decoder of an <eos>-terminated request, §8f N1): b = decode step | (eos + 1) << 12
__host__ __device__ inline int row_step(int b) { return b & 0xFFF; }
__host__ __device__ inline int row_eos(int b) { return (b >> 12) - 1; }

// Epilogue kinds (template parameter of the kernels).
enum { EPI_LSTM = 0, EPI_PROJ = 1, EPI_LEAF = 2, EPI_INTERNAL = 3 };

// Gates per cell kind and the packed ("gate-interleaved") weight layout:
//   packed row n = u * G + g  <->  paper row g * H + u   (u = hidden unit, g = gate)
// so that one tile of U units holds every gate of its units (fused epilogue, A9).
__host__ __device__ inline int gates_of(int epi) {
  return epi == EPI_LSTM ? 4 : epi == EPI_LEAF ? 3 : epi == EPI_INTERNAL ? 5 : 1;
}

struct StepArgs {
  int epi;          // EPI_*
  int G;            // gates (4 LSTM, 3 leaf, 5 internal, 1 projection)
  int H;            // hidden
  int K0, K1;       // widths of the two operand segments ([x ; h] or [h_L ; h_R]); K1 may be 0
  int U;            // hidden units per CTA tile (tile rows = G * U <= 128)
  int S;            // split-K factor = cluster size
  int kslice;       // K per CTA (multiple of 64)
  int b;            // rows in the task
  int layer;        // layer index inside the pool (0-based)
  int n_slots;      // pool slots (stride between the two h parities)
  const RowDesc* rows;
  const void* E;        // embedding [V][H] (bf16 or fp32)
  int V;
  const void* h_lower;  // pool h of layer-1, base of parity 0 ([2][n_slots][H]); layer 0: null
  void* h_pool;         // pool h of this layer ([2][n_slots][H])
  float* c_pool;        // pool c of this layer ([n_slots][H])
  int* tok;             // feed tokens [n_slots]
  const void* W;        // fp32 path: packed [rows][K]; bf16 path: stage tiles (launch_pack_tiles)
  const float* bias;    // packed bias [rows]
  int W_rows;           // G * H (or V for the projection)
  float* res_h;         // result rows [max_requests][res_layers][H]
  float* res_c;
  int res_layers;
  // projection + argmax (EPI_PROJ)
  unsigned long long* amax;   // [bmax] packed (value, ~index) keys, zero between tasks
  unsigned int* done_ctas;    // CTA completion counter for the last-CTA finalize
  int32_t* res_tok;           // [max_requests][max_decode]
  int max_decode;
  float* logits;              // debug [max_requests][max_decode][V] or null
  unsigned long long* phase;  // diagnostics: per-CTA %globaltimer at phase boundaries, or null
  int max_stages;             // experiments (BM_MAX_STAGES): cap on pipeline stages, 0 = default
  int experiment;             // diagnostics (BM_EXPERIMENT) bit 1: no activation reads (zero
                              // fill), bit 2: no weight copies; results are garbage
  // launch path
  unsigned long long* signal; // non-null on a task's last launch: host-mapped completion counter
  unsigned long long sig_value;  // the value this task's completion publishes in *signal (seq + 1)
  unsigned int* sig_ctas;     // CTA counter for the fused signal (zero between launches)
  int pdl;                    // launch with programmatic dependent launch (overlap setup)
  int cpb;                    // CTA-pair kernel: batch columns per column block
  int wcb, xring, xkb;        // ring plan (set by the launcher): K blocks per weight chunk,
                              // activation ring bytes, K blocks per activation stage
  unsigned long long* span;   // time_kernels: slot {min CTA start, CTAs done} (device memory)
  unsigned long long* span_acc;  // {sum of launch spans in ns, launches} of the launch's kernel
                                 // class (bm.h BM_K_*): the last CTA adds
  unsigned long long* span_log;  // or null: the last CTA stores this launch's span (ns) here
  const unsigned int* rows_flag;  // ring rows: published once *rows_flag >= rows_seq (or null)
  unsigned int rows_seq;
  unsigned int* dep_flag;     // launch chain: sequence number of the last completed launch
  unsigned int dep_seq;       // this launch's sequence number (waits for dep_seq - 1)
  unsigned long long* tl;     // diagnostics (BM_TIMELINE): {~first CTA start, ~first past the
                              // PDL wait, last CTA end, CTAs} in %globaltimer ns, or null
  int* dead;                  // [n_slots] 1 once the slot's request emitted <eos> (ROW_EOS rows
                              // are then no-ops); cleared by the request's first encoder step
  int* eos_host;              // host-mapped [max_requests]: decode step + 1 of the <eos>, or 0
  int pchunk;                 // split-K exchange chunk (columns), 0 = whole tile (BM_PCHUNK)
  int wcpa;                   // LSTM single-CTA kernel: weights by cp.async in the stages;
                              // CTA-pair kernel: 2 = the stage's weight part by one bulk copy
                              // of the TMA warp (completion on the stage's full barrier)
  int small_plan;             // engine has >= 2 workers: LSTM launches use a <= 113 KB shared-
                              // memory plan (no CTA pairs) so two workers' CTAs share an SM
  int cbuf_off;               // set by the launcher: shared-memory offset (from the 1 KB-aligned
                              // base) of the epilogue's prefetched c-state rows
  int wslots;                 // set by the launcher: weight ring slots (one TMA lane each)
  float* scratch;             // split-K partial exchange through L2 (cell_pair2_kernel): per CTA
                              // [128 rows][256 columns] fp32, kPairScratchCTAs regions
};

// cell_pair2_kernel's split-K scratch: regions of [128][256] fp32 for up to this many CTAs.
constexpr int kPairScratchCTAs = 148;
cudaError_t launch_pair2(StepArgs a, const RowDesc* rows_host, cudaStream_t st, bool* done);

// Completion signals (A12): a ring of host-mapped slots; task `seq` of a worker writes seq + 1
// into slot seq % kSignalSlots (one writer per slot at a time: kSignalSlots >> tasks in flight).
constexpr int kSignalSlots = 256;

// Persistent weight-stationary LSTM engine (lstm_persistent_sm100.cu).
struct TaskHdr {
  int32_t seq;      // run-local task index; the kernel polls for the value it expects
  int32_t b;        // rows; -1 = stop
  int32_t row_off;  // first row in the device descriptor ring
  int32_t flags;
};
struct PersistArgs {
  int H, K, K0, S, kslice, n_slots, res_layers, hdr_ring;
  const TaskHdr* hdr;
  const RowDesc* rows;
  const void* E;
  void* h_pool;
  float* c_pool;
  int* tok;
  const void* W;              // stage-tile layout (launch_pack_tiles)
  const float* bias;
  float* res_h;
  float* res_c;
  unsigned int* gbar;         // grid-barrier counter (zero at launch)
  int* err;                   // set to 1 if the kernel aborted (host stopped feeding)
  unsigned long long* signal; // host-mapped completion slots [kSignalSlots]
  unsigned long long sig_base;   // worker task index of the run's first task
  unsigned long long* span;   // optional: 64 task-start slots (time_kernels)
  unsigned long long* span_acc;
  unsigned long long* phase;  // diagnostics (BM_PHASE_DUMP): per-CTA timestamps of task 20
};
cudaError_t launch_lstm_persistent(const PersistArgs& a, cudaStream_t st);
int persistent_smem_bytes();

// bf16 / tcgen05 path (cell_step_sm100.cu). a.W: weights in the stage-tile layout
// (launch_pack_tiles): [tile][K/64][tile_rows][64] bf16, 128B-swizzled rows.
// Row descriptors of one launch passed by value as a kernel parameter (the launch carries them:
// no host->device copy and no cross-stream dependency between consecutive launches, so PDL
// overlaps a launch's prologue with the previous launch's tail).
constexpr int kMaxRowsInline = 512;
// rows_host: the launch's rows in host memory (b <= kMaxRowsInline) -- passed inline; or null,
// then a.rows must point to device memory holding them.
// *kclass (may be null) receives the kernel class (bm.h BM_K_*) the launch ran as; the launcher
// picks the kernel, so a.span_acc must already point at that class's accumulator: pass
// span_acc_base (the [BM_K_CLASSES][2] array) and the launcher offsets it.
cudaError_t launch_cell_step_sm100(const StepArgs& a, const RowDesc* rows_host, cudaStream_t st,
                                   int* kclass = nullptr);
// fp32 / SIMT path (cell_step_simt.cu)
cudaError_t launch_cell_step_simt(const StepArgs& a, cudaStream_t st);

// Weight preparation (load time): fp32 paper layout -> packed, gate-interleaved, bf16 or fp32.
cudaError_t launch_pack_rows(const float* src, void* dst, float* bias_dst, const float* bias_src,
                             int G, int H, int K, int bf16, cudaStream_t st);
cudaError_t launch_pack_tiles(const float* src, void* dst, int G, int H, int K, int tile_rows,
                              int n_rows, cudaStream_t st);
// act16 = 1: to the tensor-core path's fp16 activation storage (embeddings); 0: fp32 copy
cudaError_t launch_convert(const float* src, void* dst, size_t n, int act16, cudaStream_t st);
// Completion signal (A12): bump a host-mapped counter after everything before it in stream.
cudaError_t launch_signal(unsigned long long* counter, unsigned long long value, cudaStream_t st);
// Pool access helpers (tests): gather/scatter fp32 rows of h (bf16 or fp32) and c.
cudaError_t launch_pool_io(void* h_pool, float* c_pool, const int32_t* slots, int n, int H,
                           float* h_buf, float* c_buf, int write, int bf16, cudaStream_t st);

// Kernel-count bookkeeping: number of kernels one launch_* call issues.
}  // namespace bm
