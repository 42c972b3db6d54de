// scheduler.cpp -- request processor + Algorithm 1 (BatchMaker, EuroSys'18) in C++.
//
// Request processor (§4.2, §4.3, §4.4):
//   chain     -> one subgraph of L nodes (one cell type)
//   seq2seq   -> encoder subgraph (S nodes) + decoder subgraph (T nodes); the decoder is passed
//                to the scheduler when the encoder subgraph completes
//   tree      -> one subgraph per leaf + one subgraph of all internal nodes, passed on when
//                every leaf has completed
// Algorithm 1 (L345-L369): Schedule(worker) picks a cell type in three tiers, Batch forms up to
// MaxTasksToSubmit tasks, FormBatchedTask scans the type's subgraph queue in FIFO order.
// UpdateNodesDependency releases intra-subgraph successors at submission (L381); inter-subgraph
// dependencies are released when the subgraph completes (L331, L385).
//
// Readings where the paper is silent (restated in DESIGN.md) are marked
// [Sxx]. The oracle/scheduler.py replay implements the same specification independently; the
// tests compare the two task logs bit for bit.
#include <algorithm>
#include <functional>

#include "engine.h"

namespace bm {
namespace {

inline Subgraph& SG(Engine& e, int req, int sid) { return e.reqs[req].sg(sid); }

void enqueue(Engine& e, int req, int sid) {  // append to the cell type's FIFO [S18]
  Subgraph& g = SG(e, req, sid);
  Cell& c = e.cells[g.ct];
  g.queued = true;
  g.q_next_req = g.q_next_sid = -1;
  g.q_prev_req = c.q_tail_req;
  g.q_prev_sid = c.q_tail_sid;
  if (c.q_tail_req >= 0) {
    Subgraph& t = SG(e, c.q_tail_req, c.q_tail_sid);
    t.q_next_req = req;
    t.q_next_sid = sid;
  } else {
    c.q_head_req = req;
    c.q_head_sid = sid;
  }
  c.q_tail_req = req;
  c.q_tail_sid = sid;
  c.ready_nodes += static_cast<int64_t>(g.ready.size());
}

void dequeue(Engine& e, int req, int sid) {
  Subgraph& g = SG(e, req, sid);
  Cell& c = e.cells[g.ct];
  if (g.q_prev_req >= 0) {
    Subgraph& p = SG(e, g.q_prev_req, g.q_prev_sid);
    p.q_next_req = g.q_next_req;
    p.q_next_sid = g.q_next_sid;
  } else {
    c.q_head_req = g.q_next_req;
    c.q_head_sid = g.q_next_sid;
  }
  if (g.q_next_req >= 0) {
    Subgraph& n = SG(e, g.q_next_req, g.q_next_sid);
    n.q_prev_req = g.q_prev_req;
    n.q_prev_sid = g.q_prev_sid;
  } else {
    c.q_tail_req = g.q_prev_req;
    c.q_tail_sid = g.q_prev_sid;
  }
  c.ready_nodes -= static_cast<int64_t>(g.ready.size());
  g.queued = false;
}

// insert node v into the subgraph's ready list keeping (height, index) order [S18]
void make_ready(Engine& e, int req, int sid, int v) {
  Request& r = e.reqs[req];
  Subgraph& g = r.sg(sid);
  int pos = g.ready.size();
  if (r.kind == BM_REQ_TREE) {
    const std::pair<int, int> kv(r.height[v], v);
    pos = 0;
    while (pos < g.ready.size() && std::make_pair(r.height[g.ready[pos]], g.ready[pos]) < kv) ++pos;
  }
  g.ready.insert_at(pos, v);
  if (g.queued) e.cells[g.ct].ready_nodes += 1;
}

int slot_alloc(Engine& e) {  // lowest free index [S22]
  std::pop_heap(e.free_slots_heap.begin(), e.free_slots_heap.end(), std::greater<int>());
  const int s = e.free_slots_heap.back();
  e.free_slots_heap.pop_back();
  return s;
}

int slots_needed(const Request& r) { return r.kind == BM_REQ_TREE ? r.n_nodes : 1; }

}  // namespace

void slot_release(Engine& e, int s) {
  e.free_slots_heap.push_back(s);
  std::push_heap(e.free_slots_heap.begin(), e.free_slots_heap.end(), std::greater<int>());
}

bool has_ready(const Engine& e) {
  for (const auto& q : e.buckets)
    if (!q.empty()) return true;
  for (const Cell& c : e.cells)
    if (c.ready_nodes > 0) return true;
  return false;
}

// ---------------------------------------------------------------- admission (A1)
bm_status admit_request(Engine& e, int ri) {
  Request& r = e.reqs[ri];
  r.n_completed = 0;
  r.started = false;
  r.slot = -1;
  r.t_first = -1;
  r.t_done = -1;
  r.eos_step = -1;
  if (e.eos_host != nullptr) e.eos_host[ri] = 0;  // no device write can be pending: entry free
  if (e.cfg.policy == BM_POLICY_GRAPH) {  // padding + bucketing: bucket (i*w, (i+1)*w] (L427)
    const size_t i = static_cast<size_t>((r.n_nodes - 1) / e.cfg.bucket_width);
    if (e.buckets.size() <= i) e.buckets.resize(i + 1);
    e.buckets[i].push_back(ri);
    return BM_OK;
  }
  if (r.kind == BM_REQ_CHAIN || r.kind == BM_REQ_SEQ2SEQ) {
    const int S = r.kind == BM_REQ_CHAIN ? r.n_nodes : r.enc_len;
    r.sg2[0] = Subgraph();
    r.sg2[1] = Subgraph();
    Subgraph& enc = r.sg2[0];
    enc.req = ri;
    enc.sid = 0;
    enc.ct = r.cell0;
    enc.n_nodes = S;
    enc.ready.assign1(0);
    if (r.kind == BM_REQ_SEQ2SEQ) {
      Subgraph& dec = r.sg2[1];
      dec.req = ri;
      dec.sid = 1;
      dec.ct = r.cell1;
      dec.n_nodes = r.n_nodes - S;
    }
    enqueue(e, ri, 0);
  } else {
    const int n = r.n_nodes;
    r.submitted.assign(n, 0);
    r.parent.assign(n, -1);
    r.height.assign(n, 0);
    r.node_slot.assign(n, -1);
    r.node_sid.assign(n, -1);
    int n_leaves = 0;
    for (int v = 0; v < n; ++v) {
      if (r.left[v] >= 0) {
        r.parent[r.left[v]] = v;
        r.parent[r.right[v]] = v;
        r.height[v] = 1 + std::max(r.height[r.left[v]], r.height[r.right[v]]);
      } else {
        ++n_leaves;
      }
    }
    r.leaves_left = n_leaves;
    r.sgv.assign(n_leaves + (n > n_leaves ? 1 : 0), Subgraph());
    int sid = 0;
    for (int v = 0; v < n; ++v) {
      if (r.left[v] >= 0) continue;
      Subgraph& g = r.sgv[sid];
      g.req = ri;
      g.sid = sid;
      g.ct = r.cell0;
      g.n_nodes = 1;
      g.ready.assign1(v);
      r.node_sid[v] = sid;
      ++sid;
    }
    r.internal_sid = -1;
    if (n > n_leaves) {
      Subgraph& g = r.sgv[sid];
      g.req = ri;
      g.sid = sid;
      g.ct = r.cell1;
      g.n_nodes = n - n_leaves;
      g.ready.clear();
      for (int v = 0; v < n; ++v)
        if (r.left[v] >= 0) r.node_sid[v] = sid;
      r.internal_sid = sid;
    }
    for (int s = 0; s < n_leaves; ++s) enqueue(e, ri, s);
  }
  return BM_OK;
}

// ---------------------------------------------------------------- Algorithm 1
namespace {

struct Cand {
  int req, sid, node;
};

// FormBatchedTask(ct, worker), Alg. 1 lines 24-32, with the slot check [S22]. Pure.
void form_batched_task(Engine& e, int ct, int worker, std::vector<Cand>& batch) {
  batch.clear();
  Cell& c = e.cells[ct];
  const int bmax = c.d.max_batch;
  int free = static_cast<int>(e.free_slots_heap.size());
  int req = c.q_head_req, sid = c.q_head_sid;
  int last_new_req = -1;
  while (req >= 0) {                                              // line 26
    Subgraph& g = SG(e, req, sid);
    const int nreq = g.q_next_req, nsid = g.q_next_sid;
    if (g.pinned < 0 || g.pinned == worker) {                     // line 27
      Request& r = e.reqs[req];
      for (int i = 0; i < g.ready.size(); ++i) {                  // line 28
        const int v = g.ready[i];
        int need = 0;
        if (!r.started && last_new_req != req) need = slots_needed(r);
        if (need > free) break;
        free -= need;
        if (need) last_new_req = req;
        batch.push_back({req, sid, v});                           // line 29
        if (static_cast<int>(batch.size()) == bmax) return;       // lines 30-31
      }
    }
    req = nreq;
    sid = nsid;
  }
}                                                                 // line 32

void release_successor(Engine& e, int req, int sid, int v) {  // UpdateNodesDependency [S20]
  Request& r = e.reqs[req];
  if (r.kind != BM_REQ_TREE) {
    const int nxt = v + 1;
    const int end = (r.kind == BM_REQ_SEQ2SEQ && sid == 0) ? r.enc_len : r.n_nodes;
    if (nxt < end) make_ready(e, req, sid, nxt);
  } else {
    const int p = r.parent[v];
    if (p >= 0 && r.node_sid[p] == sid && !r.submitted[p] && r.submitted[r.left[p]] &&
        r.submitted[r.right[p]]) {
      if (!r.sg(sid).ready.contains(p)) make_ready(e, req, sid, p);
    }
  }
}

// Device row descriptor of a scheduled node (A3): what the kernels need to gather and scatter.
RowDesc describe_row(const Request& r, int ri, int node, int slot) {
  RowDesc d{};
  d.slot = slot;
  int flags = 0;
  if (r.kind == BM_REQ_TREE) {
    if (r.left[node] < 0) {
      d.a = r.tokens[node];
    } else {
      d.a = r.node_slot[r.left[node]];
      d.b = r.node_slot[r.right[node]];
    }
    if (node == r.n_nodes - 1) flags |= ROW_LAST;
  } else {
    const int step = node;  // global step (encoder steps then decoder steps)
    if (step == 0) flags |= ROW_FIRST;
    if (step & 1) flags |= ROW_PARITY;
    if (r.kind == BM_REQ_CHAIN || step < r.enc_len) {
      d.a = r.tokens[step];
    } else {
      const int s = step - r.enc_len;
      d.a = s == 0 ? 1 /* <go> */ : -1 /* feed previous: tok[slot] on device */;
      d.b = s;
      if (r.eos_stop) {  // N1: any step may be the last -> every step writes the result row
        flags |= ROW_EOS | ROW_LAST;
        d.b = s | ((r.eos_id + 1) << 12);
      }
    }
    if (step == r.n_nodes - 1) flags |= ROW_LAST;
  }
  d.flags = flags | (ri << 8);  // result row = request table index
  return d;
}

Task submit(Engine& e, int ct, int worker, const std::vector<Cand>& batch) {
  Task t;
  t.ct = ct;
  t.tick = e.now;
  t.worker = worker;
  t.rows.reserve(batch.size());
  t.desc.reserve(batch.size());
  Cell& c = e.cells[ct];
  for (const Cand& x : batch) {
    Request& r = e.reqs[x.req];
    if (!r.started) {  // take every slot the request will need [S22]
      r.started = true;
      if (r.kind == BM_REQ_TREE) {
        for (int u = 0; u < r.n_nodes; ++u) r.node_slot[u] = slot_alloc(e);
      } else {
        r.slot = slot_alloc(e);
      }
    }
    if (r.t_first < 0) r.t_first = e.now;
    const int slot = r.kind == BM_REQ_TREE ? r.node_slot[x.node] : r.slot;
    t.rows.push_back({x.req, x.node, slot});
    Subgraph& g = r.sg(x.sid);
    g.ready.erase_value(x.node);
    if (g.queued) c.ready_nodes -= 1;
    g.n_submitted += 1;
    if (r.kind == BM_REQ_TREE) r.submitted[x.node] = 1;
    t.desc.push_back(describe_row(r, x.req, x.node, slot));
  }
  c.running_tasks += 1;
  for (const Cand& x : batch) release_successor(e, x.req, x.sid, x.node);   // line 18
  // lines 20-21: rows of one subgraph are contiguous in a batch (FormBatchedTask walks one
  // subgraph's ready nodes at a time), so each subgraph is counted once.
  for (size_t i = 0; i < batch.size(); ++i) {
    const Cand& x = batch[i];
    if (i > 0 && batch[i - 1].req == x.req && batch[i - 1].sid == x.sid) continue;
    Subgraph& g = SG(e, x.req, x.sid);
    g.inflight += 1;
    g.pinned = worker;
    if (g.n_submitted == g.n_nodes && g.queued) dequeue(e, x.req, x.sid);
  }
  return t;
}

// Batch(ct, worker), Alg. 1 lines 12-23.
int batch_tasks(Engine& e, int ct, int worker, std::vector<Task>& out) {
  static thread_local std::vector<Cand> batch;
  int num_tasks = 0;                                                       // line 13
  while (num_tasks < e.cfg.max_tasks_to_submit) {                          // line 14
    form_batched_task(e, ct, worker, batch);                              // line 15
    if (batch.empty()) break;                                              // [S15]
    if (static_cast<int>(batch.size()) >= e.cfg.min_followon_batch || num_tasks == 0) {  // 16
      out.push_back(submit(e, ct, worker, batch));                        // lines 17-21
      ++num_tasks;                                                         // line 19
    } else {
      break;                                                               // line 23
    }
  }
  return num_tasks;
}

}  // namespace

// ---------------------------------------------------------------- graph batching (N4)
// The padding + bucketing baseline of §7.1 (L427-L437) over the same cell kernels: round robin
// over non-empty buckets [G1], a batch of <= bmax requests of one bucket runs the bucket's
// graph unrolled to (i+1)*w steps -- one task per step, same rows, padded steps on the pad
// token [G2] -- and every request of the batch completes when its last task retires.
static int schedule_graph(Engine& e, std::vector<Task>& out) {
  const int nb = static_cast<int>(e.buckets.size());
  int pick = -1;
  for (int d = 0; d < nb; ++d) {                        // cyclic scan after the last served
    const int i = (e.last_bucket + 1 + d) % nb;
    if (!e.buckets[i].empty()) {
      pick = i;
      break;
    }
  }
  if (pick < 0) return 0;
  std::deque<int>& q = e.buckets[pick];
  const int ct = e.reqs[q.front()].cell0;
  Cell& c = e.cells[ct];
  const int n = std::min<int>({c.d.max_batch, static_cast<int>(q.size()),
                               static_cast<int>(e.free_slots_heap.size())});
  if (n == 0) return 0;
  e.last_bucket = pick;
  std::vector<int> rids(n);
  for (int k = 0; k < n; ++k) {
    rids[k] = q.front();
    q.pop_front();
    Request& r = e.reqs[rids[k]];
    r.started = true;
    r.slot = slot_alloc(e);                               // [G3]
    r.t_first = e.now;
  }
  const int steps = (pick + 1) * e.cfg.bucket_width;     // the bucket's unrolled graph
  for (int s = 0; s < steps; ++s) {
    Task t;
    t.ct = ct;
    t.tick = e.now;
    t.rows.reserve(n);
    t.desc.reserve(n);
    for (int ri : rids) {
      const Request& r = e.reqs[ri];
      t.rows.push_back({ri, s, r.slot});
      RowDesc d{};
      d.slot = r.slot;
      d.a = s < r.n_nodes ? r.tokens[s] : 0;             // pad token past the request's end [G2]
      int flags = 0;
      if (s == 0) flags |= ROW_FIRST;
      if (s & 1) flags |= ROW_PARITY;
      if (s == r.n_nodes - 1) flags |= ROW_LAST;          // result row = the real last step
      d.flags = flags | (ri << 8);
      t.desc.push_back(d);
    }
    c.running_tasks += 1;
    if (s == steps - 1) t.batch_reqs = rids;
    out.push_back(std::move(t));
  }
  return steps;
}

// Schedule(worker), Alg. 1 lines 4-11. If the chosen type forms no task only because the
// slot pool is exhausted, fall through to the next choice [S22].
int schedule(Engine& e, int worker, std::vector<Task>& out) {
  if (e.cfg.policy == BM_POLICY_GRAPH) return schedule_graph(e, out);
  const int nc = static_cast<int>(e.cells.size());
  uint64_t excluded = 0;
  for (int attempt = 0; attempt < nc; ++attempt) {
    int best = -1;
    for (int tier = 0; tier < 3 && best < 0; ++tier) {
      for (int i = 0; i < nc; ++i) {
        if (excluded >> i & 1) continue;
        const Cell& c = e.cells[i];
        bool in;
        if (tier == 0) in = c.ready_nodes >= c.d.max_batch;                  // line 5 [S13]
        else if (tier == 1) in = c.running_tasks == 0 && c.ready_nodes > 0;   // line 7
        else in = c.ready_nodes > 0;                                          // line 9
        if (!in) continue;
        if (best < 0 || c.d.priority > e.cells[best].d.priority) best = i;    // line 10
      }
    }
    if (best < 0) return 0;
    const int n = batch_tasks(e, best, worker, out);                          // line 11
    if (n > 0) return n;
    excluded |= 1ull << best;
  }
  return 0;
}

// ---------------------------------------------------------------- completion (A13)
void retire_task(Engine& e, Task& t) {
  Cell& c = e.cells[t.ct];
  c.running_tasks -= 1;
  if (e.cfg.policy == BM_POLICY_GRAPH) {   // the graph returns every output at its end
    for (int ri : t.batch_reqs) {
      Request& r = e.reqs[ri];
      r.done = true;
      r.t_done = e.now;
      bm_completion cp;
      cp.req_id = r.id;
      cp.user_tag = r.tag;
      cp.t_arrival = r.t_arrival;
      cp.t_first = r.t_first;
      cp.t_done = r.t_done;
      e.completions.push_back(cp);
      e.completed_total += 1;
      slot_release(e, r.slot);
      if (!e.cfg.keep_results) {
        r.used = false;
        e.n_live_reqs -= 1;
      }
    }
    return;
  }
  for (size_t i = 0; i < t.rows.size(); ++i) {
    const TaskRow& row = t.rows[i];
    Request& r = e.reqs[row.req];
    const int sid = r.sid_of(row.node);
    Subgraph& g = r.sg(sid);
    if (r.eos_stop && r.eos_step < 0 && sid == 1) {
      // N1 (L715): did this row's decode step emit <eos>? Only the retire of the task holding
      // that step acts on it (tasks retire in order), so the replay can follow the same rule.
      const int s = row.node - r.enc_len;
      const int rep = e.device() ? static_cast<volatile int*>(e.eos_host)[row.req] - 1 : r.dry_eos_step;
      if (rep == s) {
        r.eos_step = s;
        // nothing more is submitted: the decoder ends with the nodes already in flight
        if (g.queued) dequeue(e, row.req, 1);
        g.ready.clear();
        g.n_nodes = g.n_submitted;
        r.n_nodes = r.enc_len + g.n_nodes;
      }
    }
    bool seen = false;  // rows of one subgraph are contiguous (see submit)
    if (i > 0 && t.rows[i - 1].req == row.req) {
      const TaskRow& o = t.rows[i - 1];
      seen = r.sid_of(o.node) == sid;
    }
    if (!seen) {
      g.inflight -= 1;
      if (g.inflight == 0) g.pinned = -1;   // unpin (L381)
    }
    g.n_completed += 1;
    r.n_completed += 1;
    if (g.n_completed == g.n_nodes) {       // subgraph done: inter-subgraph deps [S20]
      if (r.kind == BM_REQ_SEQ2SEQ && sid == 0 && r.sg2[1].n_nodes > 0) {
        r.sg2[1].ready.assign1(r.enc_len);
        enqueue(e, row.req, 1);
      } else if (r.kind == BM_REQ_TREE && r.left[row.node] < 0) {
        if (--r.leaves_left == 0 && r.internal_sid >= 0) {
          Subgraph& is = r.sgv[r.internal_sid];
          is.ready.clear();
          enqueue(e, row.req, r.internal_sid);
          for (int v = 0; v < r.n_nodes; ++v)
            if (r.left[v] >= 0 && r.submitted[r.left[v]] && r.submitted[r.right[v]])
              make_ready(e, row.req, r.internal_sid, v);
        }
      }
    }
    if (r.n_completed == r.n_nodes) {       // request leaves the system (L267, L331)
      r.done = true;
      r.t_done = e.now;
      bm_completion cp;
      cp.req_id = r.id;
      cp.user_tag = r.tag;
      cp.t_arrival = r.t_arrival;
      cp.t_first = r.t_first;
      cp.t_done = r.t_done;
      e.completions.push_back(cp);
      e.completed_total += 1;
      if (r.kind == BM_REQ_TREE) {
        for (int x : r.node_slot) slot_release(e, x);
      } else {
        slot_release(e, r.slot);
      }
      if (!e.cfg.keep_results) {  // the table entry is free again; the completion record stays
        r.used = false;
        e.n_live_reqs -= 1;
      }
    }
  }
}

}  // namespace bm
