// Host-side batched-CSR packing (P49 DAGs, P139 edges
// l = (u_s, u_d), P149 aggregation over in-edges l' = (u', u); tie-break keys
// are DESIGN.md R17).
//
// Graphs are concatenated in caller order.  Because every edge of graph b has
// both endpoints in [node_off[b], node_off[b+1]), the global sort by
// (dst, src, eid) places graph b's edges exactly at [edge_off[b], edge_off[b+1])
// — so each graph is sorted independently (two stable counting passes, LSD
// order: by src then by dst for the in-CSR; by dst then by src for the
// out-CSR) and graphs are processed in parallel by a small thread pool.
#include <cuda_runtime.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <condition_variable>
#include <functional>
#include <mutex>
#include <thread>
#include <vector>

#include "occu_internal.h"

namespace {

// Small pool of host output buffers: repeated packing of same-sized batches reuses
// already-faulted memory instead of paying mmap/page-fault costs on every call.  The
// buffers are page-locked when the CUDA runtime allows it (cudaHostAlloc), so the
// library's single CSR H2D copy runs at DMA speed instead of through a staging copy;
// the tag records which allocator owns the block.
std::mutex g_pool_mu;
struct PoolBuf { void *p; size_t bytes; bool pinned; };
std::vector<PoolBuf> g_pool;
std::vector<PoolBuf> g_live;          // handed out: base pointer -> allocator

void *pool_take(size_t bytes, size_t *cap) {
  std::lock_guard<std::mutex> lk(g_pool_mu);
  for (size_t i = 0; i < g_pool.size(); ++i)
    if (g_pool[i].bytes >= bytes && g_pool[i].bytes <= 2 * bytes + 4096) {
      PoolBuf b = g_pool[i];
      *cap = b.bytes;
      g_pool.erase(g_pool.begin() + i);
      g_live.push_back(b);
      return b.p;
    }
  *cap = bytes;
  void *p = nullptr;
  bool pinned = false;
  if (!getenv("OCCU_PACK_PAGEABLE") && cudaHostAlloc(&p, bytes, cudaHostAllocPortable) == cudaSuccess) {
    pinned = true;
  } else {
    cudaGetLastError();             // no device / driver: plain host memory
    p = malloc(bytes);
  }
  if (p) g_live.push_back({p, bytes, pinned});
  return p;
}

void pool_free_locked(const PoolBuf &b) {
  if (b.pinned) cudaFreeHost(b.p);
  else free(b.p);
}

// Returns the block to the pool (caller holds g_pool_mu).
void pool_give_locked(void *p) {
  for (size_t i = 0; i < g_live.size(); ++i)
    if (g_live[i].p == p) {
      const PoolBuf b = g_live[i];
      g_live.erase(g_live.begin() + i);
      if (g_pool.size() < 4) g_pool.push_back(b);
      else pool_free_locked(b);
      return;
    }
  free(p);
}

// Persistent worker pool for per-graph packing (no thread creation per call).
class PackPool {
 public:
  explicit PackPool(int n) {
    for (int t = 0; t < n; ++t) workers_.emplace_back([this] { loop(); });
  }
  ~PackPool() {
    {
      std::lock_guard<std::mutex> lk(mu_);
      stop_ = true;
    }
    cv_.notify_all();
    for (auto &w : workers_) w.join();
  }
  int size() const { return int(workers_.size()); }
  // Runs fn(i) for i in [0, n) on the pool plus the calling thread; returns when done.
  template <class F> void run(int n, F fn) {
    std::function<void(int)> f = fn;
    {
      std::lock_guard<std::mutex> lk(mu_);
      job_ = &f;
      n_ = n;
      next_ = 0;
      active_ = int(workers_.size());
      ++gen_;
    }
    cv_.notify_all();
    for (;;) {
      const int i = next_.fetch_add(1);
      if (i >= n) break;
      f(i);
    }
    std::unique_lock<std::mutex> lk(mu_);
    done_cv_.wait(lk, [this] { return active_ == 0; });
    job_ = nullptr;
  }

 private:
  void loop() {
    uint64_t seen = 0;
    for (;;) {
      std::function<void(int)> *job;
      int n;
      {
        std::unique_lock<std::mutex> lk(mu_);
        cv_.wait(lk, [&] { return stop_ || gen_ != seen; });
        if (stop_) return;
        seen = gen_;
        job = job_;
        n = n_;
      }
      for (;;) {
        const int i = next_.fetch_add(1);
        if (i >= n) break;
        (*job)(i);
      }
      std::lock_guard<std::mutex> lk(mu_);
      if (--active_ == 0) done_cv_.notify_all();
    }
  }
  std::vector<std::thread> workers_;
  std::mutex mu_;
  std::condition_variable cv_, done_cv_;
  std::function<void(int)> *job_ = nullptr;
  int n_ = 0, active_ = 0;
  std::atomic<int> next_{0};
  uint64_t gen_ = 0;
  bool stop_ = false;
};

PackPool &pack_pool() {
  static PackPool pool([] {
    unsigned hw = std::thread::hardware_concurrency();
    const char *env = getenv("OCCU_PACK_THREADS");
    if (env) hw = unsigned(atoi(env));
    if (hw < 1) hw = 1;
    return int(std::min(hw, 32u)) - 1;
  }());
  return pool;
}

struct Scratch {
  std::vector<int32_t> cnt, tmp;
};

// Stable counting sort of positions `in[0..m)` by key[in[i]] (keys in [0, n)).
void counting_pass(const int32_t *key, const int32_t *in, int32_t *out, int32_t m, int32_t n,
                   std::vector<int32_t> &cnt) {
  cnt.assign(static_cast<size_t>(n) + 1, 0);
  for (int32_t i = 0; i < m; ++i) cnt[key[in[i]] + 1]++;
  for (int32_t v = 0; v < n; ++v) cnt[v + 1] += cnt[v];
  for (int32_t i = 0; i < m; ++i) out[cnt[key[in[i]]]++] = in[i];
}

void pack_graph(const occu_graph_view &g, int32_t noff, int32_t eoff, occu_csr_batch *b,
                Scratch &s) {
  const int32_t n = g.num_nodes, m = g.num_edges;
  std::vector<int32_t> order(m), tmp(m);
  for (int32_t j = 0; j < m; ++j) order[j] = j;
  // in-CSR: key (dst, src, eid) -> stable by src, then stable by dst
  counting_pass(g.src, order.data(), tmp.data(), m, n, s.cnt);
  counting_pass(g.dst, tmp.data(), order.data(), m, n, s.cnt);
  std::vector<int32_t> in_pos_of(m);
  for (int32_t k = 0; k < m; ++k) {
    const int32_t j = order[k];
    b->in_src[eoff + k] = noff + g.src[j];
    b->in_dst[eoff + k] = noff + g.dst[j];
    b->in_eid[eoff + k] = eoff + j;
    in_pos_of[j] = eoff + k;
  }
  // in_ptr for this graph's nodes: in_ptr[noff+v] = eoff + #{dst < v}
  s.cnt.assign(static_cast<size_t>(n) + 1, 0);
  for (int32_t j = 0; j < m; ++j) s.cnt[g.dst[j] + 1]++;
  for (int32_t v = 0; v < n; ++v) s.cnt[v + 1] += s.cnt[v];
  for (int32_t v = 0; v < n; ++v) b->in_ptr[noff + v] = eoff + s.cnt[v];
  // out-CSR: key (src, dst, eid) -> stable by dst, then stable by src
  for (int32_t j = 0; j < m; ++j) order[j] = j;
  counting_pass(g.dst, order.data(), tmp.data(), m, n, s.cnt);
  counting_pass(g.src, tmp.data(), order.data(), m, n, s.cnt);
  for (int32_t k = 0; k < m; ++k) b->out_pos[eoff + k] = in_pos_of[order[k]];
  s.cnt.assign(static_cast<size_t>(n) + 1, 0);
  for (int32_t j = 0; j < m; ++j) s.cnt[g.src[j] + 1]++;
  for (int32_t v = 0; v < n; ++v) s.cnt[v + 1] += s.cnt[v];
  for (int32_t v = 0; v < n; ++v) b->out_ptr[noff + v] = eoff + s.cnt[v];
  for (int32_t v = 0; v < n; ++v) b->node_graph[noff + v] = -1;  // filled by caller
}

}  // namespace

void occu_host_batch_release(occu_csr_batch *b);

extern "C" occu_status occu_pack(const occu_graph_view *graphs, int32_t num_graphs,
                                 occu_csr_batch **out) {
  if (!out) {
    occu::set_global_error("occu_pack: out is NULL");
    return OCCU_EINVAL;
  }
  *out = nullptr;
  if (!graphs || num_graphs < 1) {
    occu::set_global_error("occu_pack: num_graphs < 1 or graphs NULL");
    return OCCU_EINVAL;
  }
  // validate + offsets (64-bit to detect overflow)
  int64_t N = 0, E = 0;
  for (int32_t b = 0; b < num_graphs; ++b) {
    const occu_graph_view &g = graphs[b];
    if (g.num_nodes < 1 || g.num_edges < 0 || (g.num_edges > 0 && (!g.src || !g.dst))) {
      occu::set_global_error("occu_pack: graph " + std::to_string(b) +
                             ": num_nodes < 1, num_edges < 0 or NULL edge arrays");
      return OCCU_EINVAL;
    }
    N += g.num_nodes;
    E += g.num_edges;
    if (N >= (int64_t(1) << 31) - 1 || E >= (int64_t(1) << 31) - 1) {
      occu::set_global_error("occu_pack: N or E >= 2^31");
      return OCCU_EINVAL;
    }
  }
  occu_csr_batch *b = static_cast<occu_csr_batch *>(calloc(1, sizeof(occu_csr_batch)));
  if (!b) return OCCU_ENOMEM;
  b->num_graphs = num_graphs;
  b->num_nodes = static_cast<int32_t>(N);
  b->num_edges = static_cast<int32_t>(E);
  // one allocation for all arrays
  const size_t B1 = num_graphs + 1, N1 = N + 1;
  const size_t total = 2 * B1 + 2 * N1 + 4 * static_cast<size_t>(E) + static_cast<size_t>(N);
  size_t cap = 0;
  int32_t *base = static_cast<int32_t *>(pool_take(std::max<size_t>(total, 1) * sizeof(int32_t), &cap));
  if (!base) {
    free(b);
    return OCCU_ENOMEM;
  }
  int32_t *q = base;
  b->node_off = q; q += B1;
  b->edge_off = q; q += B1;
  b->in_ptr = q; q += N1;
  b->out_ptr = q; q += N1;
  b->in_src = q; q += E;
  b->in_dst = q; q += E;
  b->in_eid = q; q += E;
  b->out_pos = q; q += E;
  b->node_graph = q; q += N;
  b->on_device = 0;
  b->priv = base;
  b->node_off[0] = 0;
  b->edge_off[0] = 0;
  for (int32_t i = 0; i < num_graphs; ++i) {
    b->node_off[i + 1] = b->node_off[i] + graphs[i].num_nodes;
    b->edge_off[i + 1] = b->edge_off[i] + graphs[i].num_edges;
  }
  b->in_ptr[N] = static_cast<int32_t>(E);
  b->out_ptr[N] = static_cast<int32_t>(E);
  // parallel over graphs on a persistent pool (results independent of schedule); each task
  // validates its graph first (ids in range, no self-loops) and records the first bad edge
  std::vector<int64_t> bad(num_graphs, -1);   // (edge << 1) | kind, kind 0 range, 1 self-loop
  auto one = [&](int i) {
    const occu_graph_view &g = graphs[i];
    for (int32_t j = 0; j < g.num_edges; ++j) {
      const int32_t s = g.src[j], t = g.dst[j];
      if (s < 0 || s >= g.num_nodes || t < 0 || t >= g.num_nodes) { bad[i] = int64_t(j) << 1; return; }
      if (s == t) { bad[i] = (int64_t(j) << 1) | 1; return; }
    }
    thread_local Scratch sc;
    pack_graph(g, b->node_off[i], b->edge_off[i], b, sc);
    for (int32_t v = b->node_off[i]; v < b->node_off[i + 1]; ++v) b->node_graph[v] = i;
  };
  if (E + N < 20000 || pack_pool().size() == 0) {
    for (int32_t i = 0; i < num_graphs; ++i) one(i);
  } else {
    pack_pool().run(num_graphs, one);
  }
  for (int32_t i = 0; i < num_graphs; ++i)
    if (bad[i] >= 0) {
      occu::set_global_error("occu_pack: graph " + std::to_string(i) + " edge " +
                             std::to_string(bad[i] >> 1) +
                             ((bad[i] & 1) ? ": self-loop (not a DAG)" : ": node id out of range"));
      occu_host_batch_release(b);
      return OCCU_EINVAL;
    }
  int32_t md = 0;
  for (int64_t v = 0; v < N; ++v) md = std::max(md, b->in_ptr[v + 1] - b->in_ptr[v]);
  b->max_in_degree = md;
  *out = b;
  return OCCU_OK;
}

// Host batches return their buffer to the pool (runtime frees device batches).
void occu_host_batch_release(occu_csr_batch *b) {
  std::lock_guard<std::mutex> lk(g_pool_mu);
  pool_give_locked(b->priv);
  free(b);
}
