// a6 — uneven layer-wise pipeline with phase-specific micro-batch sizes
// ("the slowest stage limits the overall pipeline throughput"; P:152 one
// worker per stage, master re-batches between phases; eq. (4) P:202-204:
// latency = all stages + (mu - 1) x slowest, mu_pre = ceil(B/eta),
// mu_dec = ceil(B/xi); eq. (7) P:214 asynchronous transfers; eqs. (15)-(16)
// contiguous partition).
//
// One process per GPU.  Stage r holds layers {l : stage_of_layer[l] == r}.
// Transfers are NCCL point-to-point over NVLink on two dedicated streams
// (send / recv), each on its own 2-rank "link" communicator (r -> r+1 mod P),
// so every communicator is driven by exactly one stream in one order and the
// ring (forward activations + last->first loop-back) cannot deadlock.
// Compute of micro-batch m+1 overlaps the transfer of micro-batch m
// (double-buffered activations, CUDA events for the dependencies).
//
// Intra-node TP (f4, P:63 / P:236): with plan.tp = T every stage is a group of T ranks running
// sq_stage_forward_tp on its shards; ring j (the ranks with TP index j) carries the replicated hidden
// states and loop-backs exactly as a plain pipeline does.
//
// Items (identical order on every rank): prefill m = 0..mu_pre-1, then decode
// t = 1..n_decode, m = 0..mu_dec-1.  The last stage writes out[b, 0] (hidden at
// the last prompt position) / out[b, t] and loops LN(hidden) back to stage 0
// as the next decode input (R13/R14).
#include <nccl.h>

#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "sq_common.cuh"

struct sq_comm {
  int nranks = 1, rank = 0;
  int tp = 1;               // mesh (sq_comm_init_mesh): ranks per stage; global rank = stage * tp + j
  bool local = false;
  ncclComm_t world = nullptr, send_comm = nullptr, recv_comm = nullptr;
  ncclComm_t tp_comm = nullptr;  // mesh: the tp ranks of this rank's stage (all-reduce of the TP stage)
  cudaStream_t s_send = nullptr, s_recv = nullptr;
};

namespace sq {
namespace {

sq_status nccl_check(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return SQ_OK;
  return fail(SQ_ENCCL, "%s: %s", what, ncclGetErrorString(r));
}

struct PlanView {
  int L, P, h1, h2, B, eta, xi, s, n_dec;
  int mu_pre, mu_dec;
  int heads, kappa, len_pre, max_len;  // attention (f3): heads 0 = stub; prefill chunk = s / kappa tokens
  int tp;                              // ranks per stage (f4)
  std::vector<int> first_layer;  // [P+1]
};

PlanView view(const sq_plan& pl) {
  PlanView v{};
  v.L = pl.n_layers; v.P = pl.n_stages; v.h1 = pl.hidden; v.h2 = pl.ffn; v.B = pl.B;
  v.eta = pl.eta; v.xi = pl.xi; v.s = pl.prompt_len; v.n_dec = pl.n_decode;
  v.mu_pre = (pl.B + pl.eta - 1) / pl.eta;
  v.mu_dec = (pl.B + pl.xi - 1) / pl.xi;
  v.heads = pl.n_heads;
  v.kappa = pl.kappa > 1 ? pl.kappa : 1;
  v.len_pre = pl.prompt_len / v.kappa;
  v.max_len = pl.prompt_len + pl.n_decode;
  v.tp = pl.tp > 1 ? pl.tp : 1;
  v.first_layer.assign(v.P + 1, v.L);
  for (int l = v.L - 1; l >= 0; --l) v.first_layer[pl.stage_of_layer[l]] = l;
  v.first_layer[v.P] = v.L;
  return v;
}

struct Ws {
  size_t stage, act, decin, lb, kv, kv_layer, total;
};

// n_layers: the layers passed (rank -1 with tp > 1: all tp shard sets, tp * n_layers entries)
Ws ws_layout(const PlanView& v, const sq_layer* layers, int n_layers, int rank) {
  Ws w{};
  size_t off = 0;
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  const int64_t tmax = std::max<int64_t>((int64_t)v.eta * v.len_pre, v.xi);
  w.stage = off; off += al(v.tp > 1 ? stage_tp_workspace_bytes(layers, n_layers, tmax)
                                   : stage_workspace_bytes(layers, n_layers, tmax));
  w.act = off;   off += 2 * al((size_t)tmax * v.h1 * 4);
  const int stage = rank < 0 ? -1 : rank / v.tp;
  const bool first = stage <= 0, last = stage < 0 || stage == v.P - 1;
  w.decin = off; if (first) off += al((size_t)v.B * v.h1 * 4);
  w.lb = off;    if (last) off += 2 * al((size_t)std::max(v.eta, v.xi) * v.h1 * 4);
  // KV cache of this rank's layers (f3): K and V fp16 [B][s + n_decode][h1 / tp] per layer
  w.kv_layer = v.heads > 0 ? al((size_t)v.B * v.max_len * (v.h1 / v.tp) * 2) : 0;
  w.kv = off;    off += (size_t)n_layers * 2 * w.kv_layer;
  w.total = off;
  return w;
}

// ---- CUDA-graph cache of decode stage calls.  A decode micro-batch re-runs the same kernels with the
// same pointers every step (stub attention: no position argument), so its launches are captured once
// (on a private stream: capture executes nothing) and replayed on the run's stream.  The key covers
// every value the launches bake in: the layers' structs (bits, shapes, pointers), the input/output
// buffers, the token count and the workspace; replays count their kernels in sq_launch_count.
struct GraphKey {
  uint64_t layers_hash;
  const void* x_in;
  const void* x_out;
  const void* ws;
  int64_t rows;
  int n_layers, dev;
  bool operator==(const GraphKey& o) const {
    return layers_hash == o.layers_hash && x_in == o.x_in && x_out == o.x_out && ws == o.ws && rows == o.rows &&
           n_layers == o.n_layers && dev == o.dev;
  }
};
struct GraphKeyHash {
  size_t operator()(const GraphKey& k) const {
    uint64_t h = k.layers_hash ^ (reinterpret_cast<uint64_t>(k.x_in) * 0x9E3779B97F4A7C15ull);
    h ^= reinterpret_cast<uint64_t>(k.x_out) + (h << 7) + (reinterpret_cast<uint64_t>(k.ws) >> 3) + (uint64_t)k.rows * 131;
    return (size_t)(h ^ (uint64_t)k.n_layers ^ ((uint64_t)k.dev << 40));
  }
};
struct CachedGraph {
  cudaGraphExec_t exec = nullptr;
  int64_t launches = 0;
};
std::mutex g_graph_mu;
std::unordered_map<GraphKey, CachedGraph, GraphKeyHash>* g_graphs = nullptr;
constexpr size_t kMaxGraphs = 256;

uint64_t hash_layers(const sq_layer* layers, int n) {
  const unsigned char* p = reinterpret_cast<const unsigned char*>(layers);
  uint64_t h = 1469598103934665603ull;
  for (size_t i = 0; i < (size_t)n * sizeof(sq_layer); ++i) h = (h ^ p[i]) * 1099511628211ull;
  return h;
}

bool graphs_enabled() {
  static int on = -1;
  if (on < 0) { const char* e = getenv("SQ_GRAPH"); on = (e && e[0] == '0') ? 0 : 1; }
  return on == 1;
}

// decode stage call through the graph cache (falls back to direct launches on any capture error);
// body(stream) issues the stage's launches, layers[0..n_layers) is everything they bake in
template <class Body>
sq_status stage_forward_graph(const sq_layer* layers, int n_layers, const float* x_in, int64_t rows, float* x_out,
                              void* ws, cudaStream_t S, int64_t* replays, Body body) {
  int dev = 0;
  cudaGetDevice(&dev);
  const GraphKey key{hash_layers(layers, n_layers), x_in, x_out, ws, rows, n_layers, dev};
  {
    std::lock_guard<std::mutex> lk(g_graph_mu);
    if (!g_graphs) g_graphs = new std::unordered_map<GraphKey, CachedGraph, GraphKeyHash>();
    auto it = g_graphs->find(key);
    if (it != g_graphs->end()) {
      if (cudaGraphLaunch(it->second.exec, S) != cudaSuccess) return cuda_check(cudaGetLastError(), "cudaGraphLaunch");
      count_launch((int)it->second.launches);
      ++*replays;
      return SQ_OK;
    }
  }
  cudaStream_t cs = nullptr;
  if (cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking) != cudaSuccess) {
    cudaGetLastError();
    return body(S);
  }
  const int64_t l0 = sq_launch_count();
  cudaGraph_t g = nullptr;
  cudaGraphExec_t ex = nullptr;
  sq_status st = SQ_OK;
  bool ok = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal) == cudaSuccess;
  if (ok) {
    st = body(cs);
    ok = cudaStreamEndCapture(cs, &g) == cudaSuccess && st == SQ_OK;
  }
  const int64_t n_launch = sq_launch_count() - l0;
  count_launch(-(int)n_launch);  // capture launched nothing
  if (ok) ok = cudaGraphInstantiate(&ex, g, 0) == cudaSuccess;
  if (g) cudaGraphDestroy(g);
  cudaStreamDestroy(cs);
  if (!ok) {
    cudaGetLastError();
    if (ex) cudaGraphExecDestroy(ex);
    return body(S);
  }
  {
    std::lock_guard<std::mutex> lk(g_graph_mu);
    if (g_graphs->size() >= kMaxGraphs) {
      for (auto& kv : *g_graphs) cudaGraphExecDestroy(kv.second.exec);
      g_graphs->clear();
    }
    (*g_graphs)[key] = CachedGraph{ex, n_launch};
  }
  if (cudaGraphLaunch(ex, S) != cudaSuccess) return cuda_check(cudaGetLastError(), "cudaGraphLaunch");
  count_launch((int)n_launch);
  ++*replays;
  return SQ_OK;
}

// ---- schedule: the op sequence of one rank (also exported as sq_pipeline_schedule)
std::vector<sq_sched_op> make_schedule(const PlanView& v, int rank) {
  // global rank = stage * tp + j; the ring of TP index j links (p, j) -> (p + 1, j)
  const int stage = rank < 0 ? -1 : rank / v.tp, j = rank < 0 ? 0 : rank % v.tp;
  auto g = [&](int q) { return q * v.tp + j; };
  const bool dist = rank >= 0 && v.P > 1;
  const bool first = !dist || stage == 0, last = !dist || stage == v.P - 1;
  std::vector<sq_sched_op> ops;
  auto op = [&](int kind, int item, int phase, int t, int slot, int peer, int64_t seq0, int64_t nseq, int64_t rows) {
    sq_sched_op o;
    o.kind = kind; o.item = item; o.phase = phase; o.t = t; o.slot = slot; o.peer = peer;
    o.seq0 = seq0; o.nseq = nseq; o.rows = rows;
    ops.push_back(o);
  };
  // loop-back messages, in the order the last stage sends them: prefill mb 0..mu_pre-1,
  // then decode (t, m) for t = 1..n_dec-1 (the last step's successor input is never used)
  const int n_lb = v.mu_pre + std::max(0, v.n_dec - 1) * v.mu_dec;
  int lb_posted = 0;
  const int n_pre = v.mu_pre * v.kappa;  // prefill items: (micro-batch m, chunk c)
  const int total = n_pre + v.n_dec * v.mu_dec;
  for (int it = 0; it < total; ++it) {
    const bool pre = it < n_pre;
    const int m = pre ? it / v.kappa : (it - n_pre) % v.mu_dec;
    const bool last_chunk = !pre || (it % v.kappa == v.kappa - 1);
    const int t = pre ? 0 : 1 + (it - n_pre) / v.mu_dec;
    const int64_t seq0 = pre ? (int64_t)m * v.eta : (int64_t)m * v.xi;
    const int64_t nseq = std::min<int64_t>(pre ? v.eta : v.xi, v.B - seq0);
    const int64_t T = pre ? nseq * v.len_pre : nseq;
    const int phase = pre ? SQ_PREFILL : SQ_DECODE;
    const int slot = it & 1;
    if (dist && first && !pre) {
      // post the loop-back receives this item needs (and every earlier one, in order)
      const int need = (t == 1) ? (int)((seq0 + nseq - 1) / v.eta) : v.mu_pre + (t - 2) * v.mu_dec + m;
      for (; lb_posted <= need && lb_posted < n_lb; ++lb_posted) {
        int64_t r0, nr;
        if (lb_posted < v.mu_pre) {
          r0 = (int64_t)lb_posted * v.eta;
          nr = std::min<int64_t>(v.eta, v.B - r0);
        } else {
          const int mm = (lb_posted - v.mu_pre) % v.mu_dec;
          r0 = (int64_t)mm * v.xi;
          nr = std::min<int64_t>(v.xi, v.B - r0);
        }
        op(SQ_OP_RECV_LB, lb_posted, phase, t, 0, g(v.P - 1), r0, nr, nr);
      }
    }
    if (dist && !first) op(SQ_OP_RECV_ACT, it, phase, t, slot, g(stage - 1), seq0, nseq, T);
    op(SQ_OP_COMPUTE, it, phase, t, slot, -1, seq0, nseq, T);
    if (!last) {
      op(SQ_OP_SEND_ACT, it, phase, t, slot, g(stage + 1), seq0, nseq, T);
    } else if (last_chunk) {
      op(SQ_OP_OUT, it, phase, t, slot, -1, seq0, nseq, nseq);
      if (t < v.n_dec) op(dist ? SQ_OP_SEND_LB : SQ_OP_LOOPBACK_LOCAL, it, phase, t, slot, dist ? g(0) : -1, seq0, nseq, nseq);
    }
  }
  return ops;
}

}  // namespace

sq_status comm_allreduce_sum_f32(sq_comm* c, float* buf, size_t count, cudaStream_t s) {
  if (!c || c->local) return fail(SQ_EINVAL, "allreduce: needs an NCCL communicator (sq_comm_init)");
  ncclComm_t cm = c->tp_comm ? c->tp_comm : c->world;
  if (!cm) return SQ_OK;  // a single rank
  return nccl_check(ncclAllReduce(buf, buf, count, ncclFloat, ncclSum, cm, s), "ncclAllReduce");
}
// size / rank of the TP group the comm's all-reduce spans (the stage's group for a mesh comm)
int comm_size(const sq_comm* c) { return !c ? 0 : c->tp_comm ? c->tp : c->nranks; }
int comm_rank(const sq_comm* c) { return !c ? -1 : c->tp_comm ? c->rank % c->tp : c->rank; }
bool comm_is_local(const sq_comm* c) { return c && c->local; }

}  // namespace sq

using namespace sq;

extern "C" {

sq_status sq_plan_check(const sq_plan* p) {
  if (!p) return fail(SQ_EINVAL, "sq_plan_check: null plan");
  if (p->n_layers < 1 || p->n_stages < 1 || p->n_stages > p->n_layers)
    return fail(SQ_EINVAL, "sq_plan_check: need 1 <= n_stages <= n_layers");
  if (p->hidden <= 0 || p->hidden % 128 || p->ffn <= 0 || p->ffn % 128 || p->group != 128)
    return fail(SQ_EINVAL, "sq_plan_check: hidden/ffn multiples of 128, group 128");
  if (!p->bits || !p->stage_of_layer) return fail(SQ_EINVAL, "sq_plan_check: null bits/stage_of_layer");
  if (p->B < 1 || p->eta < 1 || p->xi < 1 || p->xi > 32 || p->prompt_len < 1 || p->n_decode < 0)
    return fail(SQ_EINVAL, "sq_plan_check: need B,eta,s >= 1, 1 <= xi <= 32, n_decode >= 0");
  if (p->n_heads < 0 || (p->n_heads > 0 && (p->hidden % p->n_heads ||
                                            (p->hidden / p->n_heads != 64 && p->hidden / p->n_heads != 128))))
    return fail(SQ_EINVAL, "sq_plan_check: n_heads %d: head_dim hidden/n_heads must be 64 or 128", p->n_heads);
  if (p->kappa < 0 || (p->kappa > 1 && (p->n_heads == 0 || p->prompt_len % p->kappa)))
    return fail(SQ_EINVAL, "sq_plan_check: kappa %d needs attention (n_heads > 0) and prompt_len %% kappa == 0", p->kappa);
  if (p->tp < 0 || (p->tp > 1 && (p->hidden % (128 * p->tp) || p->ffn % (128 * p->tp) || p->n_heads % p->tp)))
    return fail(SQ_EINVAL, "sq_plan_check: tp %d needs hidden, ffn multiples of 128 tp and n_heads %% tp == 0", p->tp);
  // eqs. (15)-(16): u_{1,1} = 1, u_{L,N} = 1, adjacent layers on the same or next stage
  if (p->stage_of_layer[0] != 0 || p->stage_of_layer[p->n_layers - 1] != p->n_stages - 1)
    return fail(SQ_EINVAL, "sq_plan_check: first layer must be on stage 0 and last on stage n_stages-1");
  for (int l = 0; l < p->n_layers; ++l) {
    const int b = p->bits[l];
    if (b != 3 && b != 4 && b != 8 && b != 16) return fail(SQ_EINVAL, "sq_plan_check: layer %d bits %d", l, b);
    if (l > 0) {
      const int d = p->stage_of_layer[l] - p->stage_of_layer[l - 1];
      if (d != 0 && d != 1) return fail(SQ_EINVAL, "sq_plan_check: partition not contiguous at layer %d", l);
    }
  }
  return SQ_OK;
}

int64_t sq_pipeline_schedule(const sq_plan* plan, int rank, sq_sched_op* ops, int64_t max_ops) {
  if (sq_plan_check(plan) != SQ_OK || rank >= plan->n_stages * (plan->tp > 1 ? plan->tp : 1) || rank < -1) return -1;
  const std::vector<sq_sched_op> v = make_schedule(view(*plan), rank);
  if (ops) {
    const int64_t n = std::min<int64_t>(max_ops, (int64_t)v.size());
    for (int64_t i = 0; i < n; ++i) ops[i] = v[i];
  }
  return (int64_t)v.size();
}

size_t sq_comm_unique_id_bytes(void) { return sizeof(ncclUniqueId); }

sq_status sq_comm_get_unique_id(uint8_t* id_host) {
  if (!id_host) return fail(SQ_EINVAL, "sq_comm_get_unique_id: null");
  ncclUniqueId id;
  sq_status st = nccl_check(ncclGetUniqueId(&id), "ncclGetUniqueId");
  if (st) return st;
  memcpy(id_host, &id, sizeof(id));
  return SQ_OK;
}

namespace {
// P stage rings of tp ranks each (tp = 1: the plain pipeline), global rank = stage * tp + j
sq_status comm_init(sq_comm** out, const uint8_t* id_host, int P, int tp, int rank, const char* who) {
  const int nranks = P * tp;
  if (!out || !id_host || P < 1 || tp < 1 || rank < 0 || rank >= nranks) return fail(SQ_EINVAL, "%s: bad arguments", who);
  sq_comm* c = new sq_comm();
  c->nranks = nranks;
  c->rank = rank;
  c->tp = tp;
  if (nranks > 1) {
    ncclUniqueId id;
    memcpy(&id, id_host, sizeof(id));
    sq_status st = nccl_check(ncclCommInitRank(&c->world, nranks, id, rank), "ncclCommInitRank");
    if (st) { delete c; return st; }
    // One 2-rank communicator per link L_{p,j} = ((p, j) -> (p+1 mod P, j)), sender comm-rank 0 (key 0),
    // receiver comm-rank 1.  ncclCommSplit gives each rank one colour per call, and every rank sits on two
    // links of its ring (it sends on L_{p,j} and receives on L_{p-1,j}), so the links are spread over three
    // split calls with no rank twice in one call: A = even p < P-1, B = odd p, C = the wrap link L_{P-1,j}
    // when P is odd (for even P it is odd and lands in B).  Colour = j * P + p keeps the rings apart.
    // Ranks outside a call's links pass NCCL_SPLIT_NOCOLOR.
    const int p = rank / tp, j = rank % tp;
    if (P > 1) {
      auto call_of = [P](int l) { return (l == P - 1 && P % 2) ? 2 : (l % 2); };
      const int send_link = p, recv_link = (p - 1 + P) % P;
      ncclComm_t got[3] = {nullptr, nullptr, nullptr};
      for (int call = 0; call < 3; ++call) {
        int color = NCCL_SPLIT_NOCOLOR, key = 0;
        if (call_of(send_link) == call) { color = j * P + send_link; key = 0; }
        else if (call_of(recv_link) == call) { color = j * P + recv_link; key = 1; }
        if (call == 2 && P % 2 == 0) continue;  // no third call for even P (identical on every rank)
        st = nccl_check(ncclCommSplit(c->world, color, key, &got[call], nullptr), "ncclCommSplit");
        if (st) {
          for (ncclComm_t g : got) if (g) ncclCommDestroy(g);
          sq_comm_destroy(c);
          return st;
        }
      }
      c->send_comm = got[call_of(send_link)];
      c->recv_comm = got[call_of(recv_link)];
    }
    if (tp > 1) {  // the stage's TP group: colour = stage, comm-rank = TP index
      st = nccl_check(ncclCommSplit(c->world, p, j, &c->tp_comm, nullptr), "ncclCommSplit(tp)");
      if (st) { sq_comm_destroy(c); return st; }
    }
  }
  cudaStreamCreateWithFlags(&c->s_send, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&c->s_recv, cudaStreamNonBlocking);
  *out = c;
  return SQ_OK;
}
}  // namespace

sq_status sq_comm_init(sq_comm** out, const uint8_t* id_host, int nranks, int rank) {
  return comm_init(out, id_host, nranks, 1, rank, "sq_comm_init");
}

sq_status sq_comm_init_mesh(sq_comm** out, const uint8_t* id_host, int n_stages, int tp, int rank) {
  return comm_init(out, id_host, n_stages, tp, rank, "sq_comm_init_mesh");
}

sq_status sq_comm_init_local(sq_comm** out, int nstages) {
  if (!out || nstages < 1) return fail(SQ_EINVAL, "sq_comm_init_local: bad arguments");
  sq_comm* c = new sq_comm();
  c->nranks = nstages;
  c->rank = -1;
  c->local = true;
  *out = c;
  return SQ_OK;
}

sq_status sq_comm_destroy(sq_comm* c) {
  if (!c) return SQ_OK;
  if (c->send_comm) ncclCommDestroy(c->send_comm);
  if (c->recv_comm) ncclCommDestroy(c->recv_comm);
  if (c->tp_comm) ncclCommDestroy(c->tp_comm);
  if (c->world) ncclCommDestroy(c->world);
  if (c->s_send) cudaStreamDestroy(c->s_send);
  if (c->s_recv) cudaStreamDestroy(c->s_recv);
  delete c;
  return SQ_OK;
}

size_t sq_pipeline_workspace_bytes(const sq_plan* plan, const sq_layer* layers, int rank) {
  if (sq_plan_check(plan) != SQ_OK || !layers) return 0;
  PlanView v = view(*plan);
  if (rank >= v.P * v.tp || rank < -1) return 0;
  const int stage = rank < 0 ? -1 : rank / v.tp;
  const int n = rank < 0 ? v.L * v.tp : v.first_layer[stage + 1] - v.first_layer[stage];
  return ws_layout(v, layers, n, rank).total;
}

sq_status sq_pipeline_run(const sq_plan* plan, int rank, const sq_layer* layers, int n_layers, sq_comm* comm,
                          const float* x0, float* out, void* ws_dev, size_t ws_bytes, sq_run_stats* stats,
                          sq_stream_t stream_) {
  sq_status st = sq_plan_check(plan);
  if (st) return st;
  const PlanView v = view(*plan);
  const bool local = (rank < 0);
  if (local && comm && !comm->local) return fail(SQ_EINVAL, "sq_pipeline_run: rank -1 needs a local comm (or NULL)");
  const int TP = v.tp;
  const int stage = local ? -1 : rank / TP, tp_j = local ? -1 : rank % TP;
  if (!local) {
    if (rank >= v.P * TP) return fail(SQ_EINVAL, "sq_pipeline_run: rank %d >= n_stages %d x tp %d", rank, v.P, TP);
    if (v.P * TP > 1 && (!comm || comm->local || comm->nranks != v.P * TP || comm->rank != rank ||
                         comm->tp != TP || (TP > 1 && !comm->tp_comm)))
      return fail(SQ_EINVAL, "sq_pipeline_run: comm does not match (nranks %d, rank %d, tp %d)", comm ? comm->nranks : -1,
                  comm ? comm->rank : -1, comm ? comm->tp : -1);
  }
  const int my_first = local ? 0 : v.first_layer[stage];
  const int my_n = local ? v.L : v.first_layer[stage + 1] - v.first_layer[stage];
  const int n_sets = (local && TP > 1) ? TP : 1;  // shard sets passed (rank -1 of a TP plan: all of them)
  if (n_layers != my_n) return fail(SQ_EINVAL, "sq_pipeline_run: got %d layers, plan assigns %d to rank %d", n_layers, my_n, rank);
  if ((st = TP > 1 ? check_tp(layers, n_layers, TP, n_sets, "sq_pipeline_run") : check_layers(layers, n_layers, "sq_pipeline_run")))
    return st;
  for (int i = 0; i < n_layers * n_sets; ++i) {
    const int l = my_first + i % n_layers;
    if (layers[i].bits != plan->bits[l]) return fail(SQ_EINVAL, "sq_pipeline_run: layer %d bits differ from plan", l);
    if (layers[i].o.n != v.h1 || layers[i].o.k != v.h1 / TP || layers[i].fc1.n != v.h2 / TP)
      return fail(SQ_EINVAL, "sq_pipeline_run: layer shapes differ from plan (tp %d)", TP);
  }
  const bool is_first = local || stage == 0, is_last = local || stage == v.P - 1;
  if (is_first && !x0) return fail(SQ_EINVAL, "sq_pipeline_run: stage 0 needs x0");
  if (is_last && !out) return fail(SQ_EINVAL, "sq_pipeline_run: last stage needs out");
  const Ws W = ws_layout(v, layers, n_layers * n_sets, rank);
  if (!ws_dev || ws_bytes < W.total || (reinterpret_cast<uintptr_t>(ws_dev) & 255u))
    return fail(SQ_ENOMEM, "sq_pipeline_run: workspace %zu < %zu (or null / not 256-B aligned)", ws_bytes, W.total);

  cudaStream_t S = (cudaStream_t)stream_;
  uint8_t* base = static_cast<uint8_t*>(ws_dev);
  void* stage_ws = base + W.stage;
  const int64_t tmax = std::max<int64_t>((int64_t)v.eta * v.len_pre, v.xi);
  const size_t act_slot = ((size_t)tmax * v.h1 * 4 + 255) / 256 * 256;
  // attention (f3): per-layer cache pointers of this rank's layers (rank -1: all layers)
  // (TP, rank -1: set-major, entry r * n_layers + l)
  std::vector<void*> kcp, vcp;
  if (v.heads > 0) {
    for (int l = 0; l < n_layers * n_sets; ++l) {
      kcp.push_back(base + W.kv + (size_t)(2 * l) * W.kv_layer);
      vcp.push_back(base + W.kv + (size_t)(2 * l + 1) * W.kv_layer);
    }
  }
  float* act[2] = {reinterpret_cast<float*>(base + W.act), reinterpret_cast<float*>(base + W.act + act_slot)};
  float* dec_in = reinterpret_cast<float*>(base + W.decin);
  const size_t lb_slot = ((size_t)std::max(v.eta, v.xi) * v.h1 * 4 + 255) / 256 * 256;
  float* lb[2] = {reinterpret_cast<float*>(base + W.lb), reinterpret_cast<float*>(base + W.lb + lb_slot)};
  const int64_t out_rows = 1 + v.n_dec;
  const int64_t h1 = v.h1;
  const size_t stage_ws_bytes = W.act - W.stage;
  const bool dist = !local && v.P > 1;
  sq_comm* tp_comm = (!local && TP > 1) ? comm : nullptr;  // its stage's all-reduce group
  std::vector<sq_layer> tp_sets;                            // rank -1 of a TP plan: one stage's shard sets
  std::vector<sq_attn> tp_ctx(n_sets);

  const int64_t launches0 = sq_launch_count();
  cudaEvent_t ev_start, ev_pre, ev_end;
  cudaEventCreate(&ev_start); cudaEventCreate(&ev_pre); cudaEventCreate(&ev_end);
  cudaEvent_t ev_free[2], ev_lbfree[2], ev_recv[2], ev_ready, ev_lbready[2], ev_consumed, ev_dec_read;
  for (int i = 0; i < 2; ++i) {
    cudaEventCreateWithFlags(&ev_free[i], cudaEventDisableTiming);
    cudaEventCreateWithFlags(&ev_lbfree[i], cudaEventDisableTiming);
    cudaEventCreateWithFlags(&ev_recv[i], cudaEventDisableTiming);
    cudaEventCreateWithFlags(&ev_lbready[i], cudaEventDisableTiming);
  }
  cudaEventCreateWithFlags(&ev_ready, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&ev_consumed, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&ev_dec_read, cudaEventDisableTiming);
  cudaEventRecord(ev_start, S);
  if (dist) {
    cudaStreamWaitEvent(comm->s_send, ev_start, 0);
    cudaStreamWaitEvent(comm->s_recv, ev_start, 0);
  }
  int64_t bytes_sent = 0, replays = 0;
  cudaError_t ce = cudaSuccess;
  sq_status rs = SQ_OK;
  const auto host_t0 = std::chrono::steady_clock::now();
  // (no graphs around the NCCL all-reduce of a real TP rank)
  const bool use_graphs = graphs_enabled() && v.heads == 0 && !prof_enabled() && !tp_comm;

  // ---- execute this rank's schedule (sq_pipeline_schedule): one op at a time, compute on S,
  // sends on s_send, receives on s_recv, CUDA events for every cross-stream dependency.
  const std::vector<sq_sched_op> ops = make_schedule(v, rank);
  int lbslot = 0;
  bool lb_wait_pending = false;
  bool pre_marked = false;
  for (size_t oi = 0; oi < ops.size() && rs == SQ_OK && ce == cudaSuccess; ++oi) {
    const sq_sched_op& o = ops[oi];
    const bool pre = o.phase == SQ_PREFILL;
    float* buf = act[o.slot];
    if (!pre && !pre_marked) {
      cudaEventRecord(ev_pre, S);
      pre_marked = true;
    }
    switch (o.kind) {
      case SQ_OP_RECV_LB: {
        // WAR: a decode loop-back overwrites dec_in rows that earlier decode items read
        if (o.item >= v.mu_pre) cudaStreamWaitEvent(comm->s_recv, ev_dec_read, 0);
        ncclResult_t r = ncclRecv(dec_in + o.seq0 * h1, (size_t)(o.nseq * h1), ncclFloat32, 0, comm->recv_comm, comm->s_recv);
        if (r != ncclSuccess) rs = nccl_check(r, "ncclRecv(loop-back)");
        lb_wait_pending = true;
        break;
      }
      case SQ_OP_RECV_ACT: {
        cudaStreamWaitEvent(comm->s_recv, ev_free[o.slot], 0);  // previous use of the buffer finished
        ncclResult_t r = ncclRecv(buf, (size_t)(o.rows * h1), ncclFloat32, 0, comm->recv_comm, comm->s_recv);
        if (r != ncclSuccess) { rs = nccl_check(r, "ncclRecv"); break; }
        cudaEventRecord(ev_recv[o.slot], comm->s_recv);
        cudaStreamWaitEvent(S, ev_recv[o.slot], 0);
        break;
      }
      case SQ_OP_COMPUTE: {
        const float* x_in;
        const int chunk = pre ? o.item % v.kappa : 0;
        sq_attn ctx{};
        if (v.heads > 0) {
          ctx.n_heads = v.heads;
          ctx.max_len = v.max_len;
          ctx.n_seq_cache = v.B;
          ctx.seq0 = o.seq0;
          ctx.nseq = (int32_t)o.nseq;
          ctx.seq_len = pre ? v.len_pre : 1;
          ctx.pos0 = pre ? chunk * v.len_pre : v.s + o.t - 1;
        }
        if (is_first) {
          x_in = pre ? x0 + o.seq0 * v.s * h1 : dec_in + o.seq0 * h1;
          if (lb_wait_pending) {
            cudaEventRecord(ev_recv[0], comm->s_recv);
            cudaStreamWaitEvent(S, ev_recv[0], 0);
            lb_wait_pending = false;
          }
          if (dist) cudaStreamWaitEvent(S, ev_free[o.slot], 0);  // previous send from this buffer done
          if (pre && v.kappa > 1) {
            // gather the chunk's rows (sequence i, positions pos0..pos0+len-1) into the item buffer
            for (int64_t i = 0; i < o.nseq && !ce; ++i)
              ce = launch_copy_rows(x0 + ((o.seq0 + i) * v.s + (int64_t)chunk * v.len_pre) * h1, h1, v.len_pre, h1,
                                    buf + i * v.len_pre * h1, h1, S);
            x_in = buf;
          }
        } else {
          x_in = buf;
        }
        // one stage's layers [f, f + nl) on the item: plain, or TP (all shard sets of the stage for
        // rank -1, this rank's shards + the stage's all-reduce otherwise)
        auto run_stage = [&](int f, int nl, const float* xi) -> sq_status {
          if (TP == 1) {
            if (v.heads > 0) { ctx.k_cache = kcp.data() + f; ctx.v_cache = vcp.data() + f; }
            auto body = [&](cudaStream_t cs) {
              return stage_forward(layers + f, nl, o.phase, xi, o.rows, buf, nullptr, stage_ws, stage_ws_bytes, cs,
                                   v.heads > 0 ? &ctx : nullptr);
            };
            if (use_graphs && !pre) return stage_forward_graph(layers + f, nl, xi, o.rows, buf, stage_ws, S, &replays, body);
            return body(S);
          }
          const sq_layer* sets = layers + f;
          if (local) {
            tp_sets.resize((size_t)n_sets * nl);
            for (int r = 0; r < n_sets; ++r)
              for (int i = 0; i < nl; ++i) tp_sets[(size_t)r * nl + i] = layers[(size_t)r * n_layers + f + i];
            sets = tp_sets.data();
          }
          for (int r = 0; r < n_sets && v.heads > 0; ++r) {
            tp_ctx[r] = ctx;
            tp_ctx[r].n_heads = v.heads / TP;
            tp_ctx[r].k_cache = kcp.data() + (size_t)r * n_layers + f;
            tp_ctx[r].v_cache = vcp.data() + (size_t)r * n_layers + f;
          }
          auto body = [&](cudaStream_t cs) {
            return stage_forward_tp(sets, nl, n_sets, tp_comm, tp_j, o.phase, v.heads > 0 ? tp_ctx.data() : nullptr, xi,
                                    o.rows, buf, stage_ws, cs);
          };
          if (use_graphs && !pre) return stage_forward_graph(sets, nl * n_sets, xi, o.rows, buf, stage_ws, S, &replays, body);
          return body(S);
        };
        if (local) {
          const float* xi = x_in;
          for (int r = 0; r < v.P && rs == SQ_OK; ++r) {
            rs = run_stage(v.first_layer[r], v.first_layer[r + 1] - v.first_layer[r], xi);
            xi = buf;  // the "transfer" to the next stage is the buffer itself
          }
        } else {
          rs = run_stage(0, n_layers, x_in);
        }
        if (is_first && !pre && dist) cudaEventRecord(ev_dec_read, S);
        break;
      }
      case SQ_OP_SEND_ACT: {
        cudaEventRecord(ev_ready, S);
        cudaStreamWaitEvent(comm->s_send, ev_ready, 0);
        ncclResult_t r = ncclSend(buf, (size_t)(o.rows * h1), ncclFloat32, 1, comm->send_comm, comm->s_send);
        if (r != ncclSuccess) { rs = nccl_check(r, "ncclSend"); break; }
        bytes_sent += o.rows * h1 * 4;
        cudaEventRecord(ev_free[o.slot], comm->s_send);
        break;
      }
      case SQ_OP_OUT: {
        const float* src = pre ? buf + (int64_t)(v.len_pre - 1) * h1 : buf;
        const int64_t sstride = pre ? (int64_t)v.len_pre * h1 : h1;
        ce = launch_copy_rows(src, sstride, o.nseq, h1, out + (o.seq0 * out_rows + o.t) * h1, out_rows * h1, S);
        if (dist) cudaEventRecord(ev_free[o.slot], S);
        break;
      }
      case SQ_OP_LOOPBACK_LOCAL: {
        const float* src = pre ? buf + (int64_t)(v.len_pre - 1) * h1 : buf;
        const int64_t sstride = pre ? (int64_t)v.len_pre * h1 : h1;
        ce = launch_copy_rows(src, sstride, o.nseq, h1, lb[0], h1, S);
        if (!ce) ce = launch_layernorm_f32(lb[0], o.nseq, h1, dec_in + o.seq0 * h1, S);
        break;
      }
      case SQ_OP_SEND_LB: {
        const float* src = pre ? buf + (int64_t)(v.len_pre - 1) * h1 : buf;
        const int64_t sstride = pre ? (int64_t)v.len_pre * h1 : h1;
        cudaStreamWaitEvent(S, ev_lbfree[lbslot], 0);
        ce = launch_copy_rows(src, sstride, o.nseq, h1, lb[lbslot], h1, S);
        if (!ce) ce = launch_layernorm_f32(lb[lbslot], o.nseq, h1, lb[lbslot], S);
        if (ce) break;
        cudaEventRecord(ev_lbready[lbslot], S);
        cudaStreamWaitEvent(comm->s_send, ev_lbready[lbslot], 0);
        ncclResult_t r = ncclSend(lb[lbslot], (size_t)(o.nseq * h1), ncclFloat32, 1, comm->send_comm, comm->s_send);
        if (r != ncclSuccess) { rs = nccl_check(r, "ncclSend(loop-back)"); break; }
        bytes_sent += o.nseq * h1 * 4;
        cudaEventRecord(ev_lbfree[lbslot], comm->s_send);
        if (dist) cudaEventRecord(ev_free[o.slot], S);
        lbslot ^= 1;
        break;
      }
    }
  }
  if (!pre_marked) cudaEventRecord(ev_pre, S);
  if (dist && rs == SQ_OK) {
    cudaEventRecord(ev_ready, comm->s_send);
    cudaStreamWaitEvent(S, ev_ready, 0);
    cudaEventRecord(ev_consumed, comm->s_recv);
    cudaStreamWaitEvent(S, ev_consumed, 0);
  }
  cudaEventRecord(ev_end, S);
  const double host_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - host_t0).count();
  cudaError_t se = cudaEventSynchronize(ev_end);
  if (ce == cudaSuccess) ce = se;
  if (ce == cudaSuccess) ce = cudaGetLastError();
  if (stats && rs == SQ_OK && ce == cudaSuccess) {
    float tt = 0.f, tp = 0.f;
    cudaEventElapsedTime(&tt, ev_start, ev_end);
    cudaEventElapsedTime(&tp, ev_start, ev_pre);
    stats->t_total_ms = tt;
    stats->t_prefill_ms = tp;
    stats->t_decode_ms = tt - tp;
    stats->tokens_per_s = tt > 0 ? (double)v.B * (1 + v.n_dec) / (tt * 1e-3) : 0.0;
    stats->bytes_sent = bytes_sent;
    stats->gpu_launches = sq_launch_count() - launches0;
    stats->host_enqueue_ms = host_ms;
    stats->graph_replays = replays;
  }
  cudaEventDestroy(ev_start); cudaEventDestroy(ev_pre); cudaEventDestroy(ev_end);
  for (int i = 0; i < 2; ++i) {
    cudaEventDestroy(ev_free[i]); cudaEventDestroy(ev_lbfree[i]); cudaEventDestroy(ev_recv[i]); cudaEventDestroy(ev_lbready[i]);
  }
  cudaEventDestroy(ev_ready); cudaEventDestroy(ev_consumed); cudaEventDestroy(ev_dec_read);
  if (rs) return rs;
  return cuda_check(ce, "sq_pipeline_run");
}

}  // extern "C"
