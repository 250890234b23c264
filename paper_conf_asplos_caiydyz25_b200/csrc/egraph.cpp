#include <cstdlib>
#include <cstdio>
#include <chrono>
// E-graph loader: validation, CSR/CSC, strongly connected components, K_auto.
//
// Problem statement: PAPER.md:91-101 (classes m_j, nodes n_i, ch_i, pa_j, ec(i)).
// Sparse representation instead of dense matrices: PAPER.md:285-289 (Sec. 4.1).
// SCC decomposition of the NOTEARS term: PAPER.md:318 (Sec. 4.3).
// K_auto: reading S1.
#include <algorithm>
#include <cstring>

#include <exception>
#include <thread>

#include "internal.h"

namespace {
// SMOOTHE_LOAD_TIMING=1: seconds per loader phase on stderr (diagnostic)
struct LoadTimer {
  bool on = std::getenv("SMOOTHE_LOAD_TIMING") != nullptr;
  std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
  void operator()(const char* what) {
    if (!on) return;
    const auto n = std::chrono::steady_clock::now();
    std::fprintf(stderr, "[load] %-22s %.4f s\n", what, std::chrono::duration<double>(n - t).count());
    t = n;
  }
};
}  // namespace

namespace smoothe {

namespace {

// Class graph successors: j -> c for every c in ch_k, k in m_j (sorted, unique):
// duplicates dropped with a per-class stamp, then the (short) unique list sorted.
void class_successors(const HostGraph& g, std::vector<int32_t>& ptr, std::vector<int32_t>& adj) {
  ptr.assign(g.M + 1, 0);
  adj.clear();
  adj.reserve(g.child_class.size());
  std::vector<int32_t> stamp(g.M, -1);
  for (int32_t j = 0; j < g.M; ++j) {
    const size_t b = adj.size();
    for (int32_t k = g.class_ptr[j]; k < g.class_ptr[j + 1]; ++k)
      for (int32_t e = g.child_ptr[k]; e < g.child_ptr[k + 1]; ++e) {
        const int32_t c = g.child_class[e];
        if (stamp[c] != j) {
          stamp[c] = j;
          adj.push_back(c);
        }
      }
    std::sort(adj.begin() + b, adj.end());
    ptr[j + 1] = (int32_t)adj.size();
  }
}

// Condensation adjacency as CSR (component -> components of its classes'
// successors, duplicates kept: harmless for longest paths and Kahn's order).
void condensation_csr(int32_t M, int32_t nc, const std::vector<int32_t>& ptr,
                      const std::vector<int32_t>& adj, const std::vector<int32_t>& comp,
                      std::vector<int32_t>& cptr, std::vector<int32_t>& cadj) {
  cptr.assign(nc + 1, 0);
  for (int32_t j = 0; j < M; ++j)
    for (int32_t e = ptr[j]; e < ptr[j + 1]; ++e)
      if (comp[adj[e]] != comp[j]) cptr[comp[j] + 1]++;
  for (int32_t a = 0; a < nc; ++a) cptr[a + 1] += cptr[a];
  cadj.assign(cptr[nc], 0);
  std::vector<int32_t> fill(cptr.begin(), cptr.end() - 1);
  for (int32_t j = 0; j < M; ++j)
    for (int32_t e = ptr[j]; e < ptr[j + 1]; ++e)
      if (comp[adj[e]] != comp[j]) cadj[fill[comp[j]]++] = comp[adj[e]];
}

// Kosaraju: finish order on the graph, then components on the transpose.
std::vector<int32_t> kosaraju(int32_t M, const std::vector<int32_t>& ptr,
                              const std::vector<int32_t>& adj) {
  std::vector<int32_t> order;
  order.reserve(M);
  std::vector<uint8_t> seen(M, 0);
  std::vector<std::pair<int32_t, int32_t>> st;
  for (int32_t s = 0; s < M; ++s) {
    if (seen[s]) continue;
    seen[s] = 1;
    st.push_back({s, ptr[s]});
    while (!st.empty()) {
      auto& top = st.back();
      if (top.second < ptr[top.first + 1]) {
        int32_t w = adj[top.second++];
        if (!seen[w]) {
          seen[w] = 1;
          st.push_back({w, ptr[w]});
        }
      } else {
        order.push_back(top.first);
        st.pop_back();
      }
    }
  }
  // transpose
  std::vector<int32_t> tptr(M + 1, 0), tadj(adj.size());
  for (size_t e = 0; e < adj.size(); ++e) tptr[adj[e] + 1]++;
  for (int32_t j = 0; j < M; ++j) tptr[j + 1] += tptr[j];
  std::vector<int32_t> fill(tptr.begin(), tptr.end() - 1);
  for (int32_t j = 0; j < M; ++j)
    for (int32_t e = ptr[j]; e < ptr[j + 1]; ++e) tadj[fill[adj[e]]++] = j;
  std::vector<int32_t> comp(M, -1);
  std::vector<int32_t> stack;
  int32_t nc = 0;
  for (auto it = order.rbegin(); it != order.rend(); ++it) {
    if (comp[*it] >= 0) continue;
    stack.push_back(*it);
    comp[*it] = nc;
    while (!stack.empty()) {
      int32_t v = stack.back();
      stack.pop_back();
      for (int32_t e = tptr[v]; e < tptr[v + 1]; ++e)
        if (comp[tadj[e]] < 0) {
          comp[tadj[e]] = nc;
          stack.push_back(tadj[e]);
        }
    }
    ++nc;
  }
  return comp;
}

// K_auto (S1): longest path from the root's component in the condensation of
// the class graph (components contracted, one hop per inter-component edge).
// Memoised DFS over the condensation from the root component.
int32_t k_auto(const HostGraph& g, const std::vector<int32_t>& ptr, const std::vector<int32_t>& adj,
               const std::vector<int32_t>& comp) {
  int32_t nc = 0;
  for (int32_t c : comp) nc = std::max(nc, c + 1);
  // condensation adjacency (duplicates are harmless for a longest path)
  std::vector<int32_t> cptr, cadj;
  condensation_csr(g.M, nc, ptr, adj, comp, cptr, cadj);
  // height(a) = longest path starting at a; the answer is height(root component)
  std::vector<int32_t> height(nc, -1);
  std::vector<std::pair<int32_t, int32_t>> st;
  const int32_t r = comp[g.root];
  st.push_back({r, cptr[r]});
  height[r] = -2;  // in progress
  while (!st.empty()) {
    auto& top = st.back();
    if (top.second < cptr[top.first + 1]) {
      const int32_t b = cadj[top.second++];
      if (height[b] == -1) {
        height[b] = -2;
        st.push_back({b, cptr[b]});
      }
    } else {
      int32_t h = 0;
      for (int32_t e = cptr[top.first]; e < cptr[top.first + 1]; ++e)
        h = std::max(h, height[cadj[e]] + 1);
      height[top.first] = h;
      st.pop_back();
    }
  }
  return height[r];
}

}  // namespace

void build_host_graph(int32_t M, int32_t N, const int32_t* class_ptr, const int64_t* child_ptr,
                      const int32_t* child_class, int32_t root, HostGraph& g) {
  LoadTimer lt;
  SM_REQUIRE(class_ptr && child_ptr && (child_class || child_ptr[N] == 0), SMOOTHE_E_INVALID_ARG,
             "NULL e-graph array");
  SM_REQUIRE(M > 0 && N > 0, SMOOTHE_E_INVALID_ARG, "num_classes and num_nodes must be > 0");
  SM_REQUIRE(N < (1 << 29), SMOOTHE_E_INVALID_ARG, "num_nodes must be < 2^29");
  SM_REQUIRE(root >= 0 && root < M, SMOOTHE_E_BAD_GRAPH, "root class out of range");
  SM_REQUIRE(class_ptr[0] == 0 && class_ptr[M] == N, SMOOTHE_E_BAD_GRAPH,
             "class_ptr must start at 0 and end at num_nodes");
  for (int32_t j = 0; j < M; ++j)
    SM_REQUIRE(class_ptr[j + 1] > class_ptr[j], SMOOTHE_E_BAD_GRAPH,
               "class " + std::to_string(j) + " is empty or class_ptr is not increasing");
  SM_REQUIRE(child_ptr[0] == 0, SMOOTHE_E_BAD_GRAPH, "child_ptr[0] must be 0");
  for (int32_t i = 0; i < N; ++i)
    SM_REQUIRE(child_ptr[i + 1] >= child_ptr[i], SMOOTHE_E_BAD_GRAPH, "child_ptr not monotone");
  SM_REQUIRE(child_ptr[N] < ((int64_t)1 << 31), SMOOTHE_E_INVALID_ARG, "more than 2^31-1 edges");
  for (int64_t e = 0; e < child_ptr[N]; ++e)
    SM_REQUIRE(child_class[e] >= 0 && child_class[e] < M, SMOOTHE_E_BAD_GRAPH,
               "child class id out of range");

  g = HostGraph();
  g.M = M;
  g.N = N;
  g.root = root;
  g.class_ptr.assign(class_ptr, class_ptr + M + 1);
  g.ec.resize(N);
  for (int32_t j = 0; j < M; ++j) {
    for (int32_t i = class_ptr[j]; i < class_ptr[j + 1]; ++i) g.ec[i] = j;
    g.max_class_size = std::max(g.max_class_size, class_ptr[j + 1] - class_ptr[j]);
  }
  lt("validate");
  // CSR children as sets
  g.child_ptr.assign(N + 1, 0);
  g.child_class.reserve(child_ptr[N]);
  std::vector<int32_t> buf;
  for (int32_t i = 0; i < N; ++i) {
    buf.assign(child_class + child_ptr[i], child_class + child_ptr[i + 1]);
    std::sort(buf.begin(), buf.end());
    buf.erase(std::unique(buf.begin(), buf.end()), buf.end());
    g.child_class.insert(g.child_class.end(), buf.begin(), buf.end());
    g.child_ptr[i + 1] = (int32_t)g.child_class.size();
  }
  g.E = (int64_t)g.child_class.size();
  lt("csr children");
  // CSC parents, by increasing e-node id
  g.par_ptr.assign(M + 1, 0);
  for (int32_t c : g.child_class) g.par_ptr[c + 1]++;
  for (int32_t j = 0; j < M; ++j) {
    g.max_in_degree = std::max(g.max_in_degree, g.par_ptr[j + 1]);
    g.par_ptr[j + 1] += g.par_ptr[j];
  }
  g.par_node.resize(g.E);
  g.par_class.resize(g.E);
  {
    std::vector<int32_t> fill(g.par_ptr.begin(), g.par_ptr.end() - 1);
    for (int32_t i = 0; i < N; ++i)
      for (int32_t e = g.child_ptr[i]; e < g.child_ptr[i + 1]; ++e) {
        int32_t slot = fill[g.child_class[e]]++;
        g.par_node[slot] = i;
        g.par_class[slot] = g.ec[i];
      }
  }

  lt("csc parents");
  // strongly connected components of the class graph
  std::vector<int32_t> sptr, sadj;
  class_successors(g, sptr, sadj);
  g.cls_child_ptr = sptr;
  g.cls_child = sadj;
  lt("scc");
  // The analysis below runs in two threads: (A) hmax, components, penalty
  // slots, K_auto and the decode levels; (B, this thread) padded layouts,
  // class edges, dmin and the padded parent lists.  They write disjoint
  // fields of g and only read the CSR / CSC arrays built above; the reverse
  // items need both (hmax, dmin) and run after the join.
  std::exception_ptr thread_error;
  std::thread thread_a([&]() {
    try {
  // hmax_j: the longest walk from class j in the class graph, i.e. the
  // largest L with g_q^{K-L}_j possibly non-zero in the reverse sweeps
  // (INT32_MAX when j can reach a cycle).  Kahn's algorithm on out-degrees:
  // a class is final once all its child classes are; classes on or above a
  // cycle never are.
  {
    std::vector<int32_t> outdeg(M), pptr(M + 1, 0), padj(sadj.size()), ready;
    for (int32_t j = 0; j < M; ++j) {
      outdeg[j] = sptr[j + 1] - sptr[j];
      for (int32_t e = sptr[j]; e < sptr[j + 1]; ++e) pptr[sadj[e] + 1]++;
    }
    for (int32_t j = 0; j < M; ++j) pptr[j + 1] += pptr[j];
    {
      std::vector<int32_t> fill(pptr.begin(), pptr.end() - 1);
      for (int32_t j = 0; j < M; ++j)
        for (int32_t e = sptr[j]; e < sptr[j + 1]; ++e) padj[fill[sadj[e]]++] = j;
    }
    g.hmax.assign(M, INT32_MAX);
    for (int32_t j = 0; j < M; ++j)
      if (outdeg[j] == 0) {
        g.hmax[j] = 0;
        ready.push_back(j);
      }
    for (size_t r = 0; r < ready.size(); ++r) {
      const int32_t c = ready[r];
      for (int32_t e = pptr[c]; e < pptr[c + 1]; ++e) {
        const int32_t j = padj[e];
        if (--outdeg[j] == 0) {
          int32_t h = 0;
          for (int32_t f = sptr[j]; f < sptr[j + 1]; ++f) h = std::max(h, g.hmax[sadj[f]] + 1);
          g.hmax[j] = h;
          ready.push_back(j);
        }
      }
    }
  }
  std::vector<int32_t> comp = kosaraju(M, sptr, sadj);
  int32_t ncomp = 0;
  for (int32_t c : comp) ncomp = std::max(ncomp, c + 1);
  std::vector<int32_t> csize(ncomp, 0);
  for (int32_t c : comp) csize[c]++;
  std::vector<uint8_t> selfloop(M, 0);
  for (int32_t j = 0; j < M; ++j)
    for (int32_t e = sptr[j]; e < sptr[j + 1]; ++e)
      if (sadj[e] == j) selfloop[j] = 1;
  std::vector<int32_t> remap(ncomp, -1);
  g.scc_of_class.assign(M, -1);
  g.scc_local.assign(M, -1);
  for (int32_t j = 0; j < M; ++j) {
    int32_t c = comp[j];
    if (csize[c] == 1 && !selfloop[j]) continue;
    if (remap[c] < 0) remap[c] = g.num_scc++;
    g.scc_of_class[j] = remap[c];
  }
  g.scc_class_ptr.assign(g.num_scc + 1, 0);
  for (int32_t j = 0; j < M; ++j)
    if (g.scc_of_class[j] >= 0) g.scc_class_ptr[g.scc_of_class[j] + 1]++;
  for (int32_t s = 0; s < g.num_scc; ++s) {
    g.scc_max = std::max(g.scc_max, g.scc_class_ptr[s + 1]);
    g.scc_class_ptr[s + 1] += g.scc_class_ptr[s];
  }
  g.scc_classes = g.scc_class_ptr[g.num_scc];
  g.scc_class.resize(g.scc_classes);
  {
    std::vector<int32_t> fill(g.scc_class_ptr.begin(), g.scc_class_ptr.end() - 1);
    for (int32_t j = 0; j < M; ++j) {
      int32_t s = g.scc_of_class[j];
      if (s < 0) continue;
      g.scc_local[j] = fill[s] - g.scc_class_ptr[s];
      g.scc_class[fill[s]++] = j;
    }
  }
  // Abar entries and penalty slots per component
  g.ent_ptr.assign(1, 0);
  g.ent_node_ptr.assign(1, 0);
  g.slot_ptr.assign(1, 0);
  g.slot_jptr.assign(1, 0);
  g.node_slot.assign(N, -1);
  std::vector<std::pair<int64_t, int32_t>> pairs;  // ((i_local, j_local), node)
  for (int32_t s = 0; s < g.num_scc; ++s) {
    pairs.clear();
    for (int32_t l = g.scc_class_ptr[s]; l < g.scc_class_ptr[s + 1]; ++l) {
      int32_t i = g.scc_class[l];
      int32_t il = g.scc_local[i];
      for (int32_t k = g.class_ptr[i]; k < g.class_ptr[i + 1]; ++k) {
        g.node_slot[k] = (int32_t)g.slot_node.size();
        g.slot_node.push_back(k);
        g.slot_iloc.push_back(il);
        for (int32_t e = g.child_ptr[k]; e < g.child_ptr[k + 1]; ++e) {
          int32_t c = g.child_class[e];
          if (g.scc_of_class[c] != s) continue;
          g.slot_jloc.push_back(g.scc_local[c]);
          pairs.push_back({((int64_t)il << 32) | (uint32_t)g.scc_local[c], k});
        }
        g.slot_jptr.push_back((int32_t)g.slot_jloc.size());
      }
    }
    g.slot_ptr.push_back((int32_t)g.slot_node.size());
    std::sort(pairs.begin(), pairs.end());
    for (size_t a = 0; a < pairs.size();) {
      size_t b = a;
      while (b < pairs.size() && pairs[b].first == pairs[a].first) {
        g.ent_node.push_back(pairs[b].second);
        ++b;
      }
      g.ent_i.push_back((int32_t)(pairs[a].first >> 32));
      g.ent_j.push_back((int32_t)(pairs[a].first & 0xffffffff));
      g.ent_node_ptr.push_back((int32_t)g.ent_node.size());
      a = b;
    }
    g.ent_ptr.push_back((int32_t)g.ent_i.size());
    if (g.scc_class_ptr[s + 1] - g.scc_class_ptr[s] > kSmallScc) {
      int32_t mx = 1;
      for (int32_t l = g.slot_ptr[s]; l < g.slot_ptr[s + 1]; ++l)
        mx = std::max(mx, g.slot_jptr[l + 1] - g.slot_jptr[l]);
      int32_t sq = 1;  // ceil(log2 mx) + 1
      while ((1 << (sq - 1)) < mx) ++sq;
      g.big_scc.push_back(s);
      g.big_scc_sq.push_back(sq);
    }
  }
  g.K_auto = k_auto(g, sptr, sadj, comp);

  // decode schedule: condensation levels reachable from the root (Kahn order)
  {
    std::vector<int32_t> cptr, cadj;
    condensation_csr(M, ncomp, sptr, sadj, comp, cptr, cadj);
    std::vector<uint8_t> seen(ncomp, 0);
    std::vector<int32_t> stack{comp[root]};
    seen[comp[root]] = 1;
    while (!stack.empty()) {
      const int32_t a = stack.back();
      stack.pop_back();
      for (int32_t e = cptr[a]; e < cptr[a + 1]; ++e)
        if (!seen[cadj[e]]) {
          seen[cadj[e]] = 1;
          stack.push_back(cadj[e]);
        }
    }
    std::vector<int32_t> indeg(ncomp, 0), depth(ncomp, -1), order;
    for (int32_t a = 0; a < ncomp; ++a)
      if (seen[a])
        for (int32_t e = cptr[a]; e < cptr[a + 1]; ++e) indeg[cadj[e]]++;
    order.push_back(comp[root]);
    depth[comp[root]] = 0;
    for (size_t i = 0; i < order.size(); ++i) {
      const int32_t a = order[i];
      for (int32_t e = cptr[a]; e < cptr[a + 1]; ++e) {
        const int32_t b = cadj[e];
        depth[b] = std::max(depth[b], depth[a] + 1);
        if (--indeg[b] == 0) order.push_back(b);
      }
    }
    for (int32_t d : depth) g.num_levels = std::max(g.num_levels, d + 1);
    g.lvl_cptr.assign(g.num_levels + 1, 0);
    g.lvl_sptr.assign(g.num_levels + 1, 0);
    for (int32_t j = 0; j < M; ++j)
      if (depth[comp[j]] >= 0) g.lvl_cptr[depth[comp[j]] + 1]++;
    for (int32_t s = 0; s < g.num_scc; ++s) {
      const int32_t d = depth[comp[g.scc_class[g.scc_class_ptr[s]]]];
      if (d >= 0) g.lvl_sptr[d + 1]++;
    }
    for (int32_t L = 0; L < g.num_levels; ++L) {
      g.lvl_cptr[L + 1] += g.lvl_cptr[L];
      g.lvl_sptr[L + 1] += g.lvl_sptr[L];
    }
    g.lvl_class.resize(g.lvl_cptr[g.num_levels]);
    g.lvl_scc.resize(g.lvl_sptr[g.num_levels]);
    std::vector<int32_t> cf(g.lvl_cptr.begin(), g.lvl_cptr.end() - 1);
    std::vector<int32_t> sf(g.lvl_sptr.begin(), g.lvl_sptr.end() - 1);
    for (int32_t j = 0; j < M; ++j)
      if (depth[comp[j]] >= 0) g.lvl_class[cf[depth[comp[j]]]++] = j;
    for (int32_t s = 0; s < g.num_scc; ++s) {
      const int32_t d = depth[comp[g.scc_class[g.scc_class_ptr[s]]]];
      if (d >= 0) g.lvl_scc[sf[d]++] = s;
    }
  }

    } catch (...) {
      thread_error = std::current_exception();
    }
  });
  struct Joiner {
    std::thread& t;
    ~Joiner() {
      if (t.joinable()) t.join();
    }
  } joiner{thread_a};

  // padded sweep layouts (multiples of 4 entries per list)
  g.pad_child_ptr.assign(N + 1, 0);
  for (int32_t i = 0; i < N; ++i) {
    const int32_t n = g.child_ptr[i + 1] - g.child_ptr[i];
    g.pad_child_ptr[i + 1] = g.pad_child_ptr[i] + ((n + 3) & ~3);
  }
  g.pad_child.assign(g.pad_child_ptr[N], root);
  g.pad_batch_node.resize(g.pad_child_ptr[N] / 4);
  for (int32_t i = 0; i < N; ++i) {
    std::copy(g.child_class.begin() + g.child_ptr[i], g.child_class.begin() + g.child_ptr[i + 1],
              g.pad_child.begin() + g.pad_child_ptr[i]);
    for (int32_t b = g.pad_child_ptr[i] / 4; b < g.pad_child_ptr[i + 1] / 4; ++b)
      g.pad_batch_node[b] = i;
  }
  lt("padded layouts");
  // class-edge index of every padded child slot (W rows of the frozen sweeps):
  // per class, pos[child class] = its index in the class's successor list
  g.pad_cedge.assign(g.pad_child_ptr[N], -1);
  {
    std::vector<int32_t> pos(M, -1);
    for (int32_t c = 0; c < M; ++c) {
      for (int32_t e = g.cls_child_ptr[c]; e < g.cls_child_ptr[c + 1]; ++e) pos[g.cls_child[e]] = e;
      for (int32_t i = g.class_ptr[c]; i < g.class_ptr[c + 1]; ++i)
        for (int32_t q = g.child_ptr[i]; q < g.child_ptr[i + 1]; ++q) {
          const int32_t e = pos[g.child_class[q]];
          SM_REQUIRE(e >= g.cls_child_ptr[c] && e < g.cls_child_ptr[c + 1] &&
                         g.cls_child[e] == g.child_class[q],
                     SMOOTHE_E_BAD_GRAPH, "internal: class successor list misses a child");
          g.pad_cedge[g.pad_child_ptr[i] + (q - g.child_ptr[i])] = e;
        }
    }
  }
  {
    const size_t nce = g.cls_child.size();
    g.cedge_class.assign(nce, 0);
    for (int32_t c = 0; c < M; ++c)
      for (int32_t e = g.cls_child_ptr[c]; e < g.cls_child_ptr[c + 1]; ++e) g.cedge_class[e] = c;
    g.cedge_ptr.assign(nce + 1, 0);
    for (int32_t i = 0; i < N; ++i)
      for (int32_t q = g.pad_child_ptr[i]; q < g.pad_child_ptr[i + 1]; ++q)
        if (g.pad_cedge[q] >= 0) g.cedge_ptr[g.pad_cedge[q] + 1]++;
    for (size_t e = 0; e < nce; ++e) g.cedge_ptr[e + 1] += g.cedge_ptr[e];
    g.cedge_node.assign(g.cedge_ptr[nce], 0);
    std::vector<int32_t> fill(g.cedge_ptr.begin(), g.cedge_ptr.end() - 1);
    for (int32_t i = 0; i < N; ++i)  // ascending e-node ids per class edge
      for (int32_t q = g.pad_child_ptr[i]; q < g.pad_child_ptr[i + 1]; ++q)
        if (g.pad_cedge[q] >= 0) g.cedge_node[fill[g.pad_cedge[q]]++] = i;
  }
  g.witem.clear();
  g.wmulti.clear();
  g.wmulti_ptr.assign(1, 0);
  g.w_num_slots = 0;
  for (int32_t c = 0; c < M; ++c) {
    const int32_t e0 = g.cls_child_ptr[c], e1 = g.cls_child_ptr[c + 1];
    if (e1 - e0 <= kWChunk) {
      g.witem.insert(g.witem.end(), {c, e0, e1, -1});
      continue;
    }
    for (int32_t e = e0; e < e1; e += kWChunk)
      g.witem.insert(g.witem.end(), {c, e, std::min(e1, e + kWChunk), g.w_num_slots++});
    g.wmulti.push_back(c);
    g.wmulti_ptr.push_back(g.w_num_slots);
  }
  lt("cedges+witems");
  // dmin_j: BFS depth of class j from the root over class -> child-class
  // edges (unreachable: INT32_MAX).  q^t_j is exactly 0 for t < dmin_j (q^0 =
  // e_root and each sweep extends the support by one edge), so the sweeps skip
  // such classes (activity windows).
  g.dmin.assign(M, INT32_MAX);
  {
    std::vector<int32_t> frontier{root}, next;
    g.dmin[root] = 0;
    for (int32_t d = 1; !frontier.empty(); ++d) {
      next.clear();
      for (int32_t j : frontier)
        for (int32_t k = g.class_ptr[j]; k < g.class_ptr[j + 1]; ++k)
          for (int32_t e = g.child_ptr[k]; e < g.child_ptr[k + 1]; ++e) {
            const int32_t c = g.child_class[e];
            if (g.dmin[c] == INT32_MAX) {
              g.dmin[c] = d;
              next.push_back(c);
            }
          }
      frontier.swap(next);
    }
  }

  g.big_class.clear();
  for (int32_t j = 0; j < M; ++j)
    if (g.class_ptr[j + 1] - g.class_ptr[j] > kBigClass) g.big_class.push_back(j);
  std::stable_sort(g.big_class.begin(), g.big_class.end(), [&](int32_t a, int32_t b) {
    return g.class_ptr[a + 1] - g.class_ptr[a] > g.class_ptr[b + 1] - g.class_ptr[b];
  });

  lt("dmin");
  // pad parents (thread B) before the join
  g.pad_par_ptr.assign(M + 1, 0);
  for (int32_t j = 0; j < M; ++j) {
    const int32_t n = g.par_ptr[j + 1] - g.par_ptr[j];
    g.pad_par_ptr[j + 1] = g.pad_par_ptr[j] + ((n + 3) & ~3);
  }
  g.pad_par.resize(2 * (size_t)g.pad_par_ptr[M]);
  for (int32_t j = 0; j < M; ++j)
    for (int32_t s = g.pad_par_ptr[j], e = g.par_ptr[j]; s < g.pad_par_ptr[j + 1]; ++s, ++e) {
      const bool real = e < g.par_ptr[j + 1];
      g.pad_par[2 * (size_t)s] = real ? g.par_node[e] : N;
      g.pad_par[2 * (size_t)s + 1] = real ? g.par_class[e] : root;
    }
  thread_a.join();
  if (thread_error) std::rethrow_exception(thread_error);
  lt("join (components, levels)");
  // reverse-sweep work items: runs of <= kRevChunk batches of one class, cut at
  // e-node boundaries; an e-node with more batches is cut into pieces of its own
  {
    // measured (C2-C5): 8 batches when the whole sweep is a few batches per
    // resident warp, 32 on the large graphs; ~8K warps are resident on a B200
    const int64_t total = g.pad_child_ptr[N] / 4;
    int32_t c = SMOOTHE_REV_CHUNK;
    if (c <= 0) c = total >= 32 * 8192 ? 32 : total >= 16 * 8192 ? 16 : 8;
    g.rev_chunk = c;
  }
  const int32_t kRevChunk = g.rev_chunk;
  g.rev_item.clear();
  g.rev_class_item_ptr.assign(M + 1, 0);
  g.rev_num_slots = 0;
  for (int32_t j = 0; j < M; ++j) {
    const int32_t cb0 = g.pad_child_ptr[g.class_ptr[j]] / 4, cb1 = g.pad_child_ptr[g.class_ptr[j + 1]] / 4;
    const size_t first = g.rev_item.size();
    auto emit = [&](int32_t b0, int32_t b1, int32_t piece) {
      const int32_t k0 = b0 < b1 ? g.pad_batch_node[b0] : -1;
      const int32_t k1 = b0 < b1 ? g.pad_batch_node[b1 - 1] : -1;
      g.rev_item.insert(g.rev_item.end(), {j, b0, b1, piece, k0, k1, g.dmin[j], g.hmax[j]});
    };
    if (cb1 - cb0 <= kRevChunk) {
      emit(cb0, cb1, 0);
    } else {
      int32_t cur = cb0;
      for (int32_t k = g.class_ptr[j]; k < g.class_ptr[j + 1]; ++k) {
        const int32_t nb0 = g.pad_child_ptr[k] / 4, nb1 = g.pad_child_ptr[k + 1] / 4;
        if (nb1 - nb0 > kRevChunk) {
          if (cur < nb0) emit(cur, nb0, 0);
          for (int32_t b = nb0; b < nb1; b += kRevChunk) emit(b, std::min(nb1, b + kRevChunk), 1);
          cur = nb1;
        } else if (nb1 - cur > kRevChunk) {
          emit(cur, nb0, 0);
          cur = nb0;
        }
      }
      if (cur < cb1) emit(cur, cb1, 0);
    }
    const int32_t n = (int32_t)((g.rev_item.size() - first) / 8);
    if (n == 1) {
      g.rev_item[first + 3] = -1;  // single item: writes its class's outputs directly
    } else {
      for (int32_t t = 0; t < n; ++t) {
        int32_t& info = g.rev_item[first + 8 * t + 3];
        info = (g.rev_num_slots++ << 1) | info;
      }
    }
    g.rev_class_item_ptr[j + 1] = g.rev_class_item_ptr[j] + n;
  }
  lt("rev items");
}

}  // namespace smoothe
