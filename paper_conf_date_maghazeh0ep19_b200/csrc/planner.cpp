// Cache-budgeted partitioner (Alg. 2 ClusterTile) and interleaver /
// emitter — SURVEY §8(a) a4, a5, a12.
//
// The whole kernel chain is one cluster (node partitioning, Alg. 1, is the
// §8(f) f1 row).  Alg. 2 is followed in the paper's order with the readings A11–A19
// (DESIGN.md §2):
//   l.4   one next unassigned block per leaf node, (x, y, z) linear order (A12);
//   l.6   FindAllDeps: transitive closure over producers, assigned blocks skipped (A13);
//   l.11  FindMoreBlks: unassigned blocks of non-source nodes whose non-empty dep set is
//         inside toBeAssigned U assigned, to a fixpoint (A14) — computed with a worklist
//         over the consumers of newly added blocks (readiness only changes when a dep
//         is added, so the fixpoint set is the same);
//   l.13  CheckCacheConst: 128 * |lines(toBeAssigned)| <= budget (A11), lines counted
//         incrementally in per-buffer bitmaps;
//   l.15  newSubKBlks <- toBeAssigned (it is always a prefix of the toBeAssigned list);
//   l.17–24 commit one sub-kernel per node in topological order (A17), drop the blocks
//         of the failing iteration (A15), INF -> KTILER_E_UNTILEABLE (A18);
//   end   when no leaf block is left, commit newSubKBlks (A16).
// Scale: O(blocks x deps) time and one byte per block + one bit per memory line, so
// 64 x 8K frames (2.6 M blocks) or a 65536^2 image plan in well under a second.
#include <algorithm>
#include <climits>
#include <cstdint>
#include <chrono>
#include <cmath>

#include "kt_internal.h"

namespace kt {

namespace {

struct Partitioner {
  const Graph& g;
  int64_t budget_lines;  // BUDGET: line cap; ROWS: -1
  int64_t rows_cap;      // ROWS: max leaf blocks per fragment
  bool force_minimal;

  std::vector<uint8_t> st;  // 0 unassigned, 1 toBeAssigned, 2 assigned
  std::vector<int64_t> tba;
  size_t new_len = 0;
  std::vector<std::vector<uint64_t>> bits;
  std::vector<std::pair<int32_t, int64_t>> dirty;
  int64_t nlines = 0, new_lines = 0;
  int64_t leaf_in_tba = 0, new_leaf = 0;
  std::vector<uint8_t> leaf_node;
  std::vector<int> leaves;
  std::vector<int64_t> cursor, scan;
  std::vector<int64_t> work;
  Schedule& out;
  int64_t nfrag = 0;

  std::vector<uint8_t> counted;  // per buffer: do its lines count against the budget
  std::vector<uint8_t> in_c;     // per node: member of the cluster being tiled
  int32_t cluster_id = 0;
  double cost = 0;               // CO_i (PAPER.md:305 l.19): sum of ET over committed sub-kernels
  bool use_et = false;

  Partitioner(const Graph& G, Schedule& o, bool resident_only) : g(G), out(o) {
    in_c.assign(g.nodes.size(), 1);
    counted.assign(g.bufs.size(), 1);
    if (resident_only) {  // only intermediates: written by one node and read by another
      std::vector<uint8_t> w(g.bufs.size(), 0), r(g.bufs.size(), 0);
      for (auto& n : g.nodes)
        for (auto& a : n.acc) (a.mode == KTILER_WRITE ? w : r)[a.buf] = 1;
      for (size_t b = 0; b < g.bufs.size(); ++b) counted[b] = w[b] && r[b];
    }
  }

  int node_of(int64_t gid) const {
    int v = 0;
    while (v + 1 < (int)g.nodes.size() && g.nodes[v + 1].gid0 <= gid) ++v;
    return v;
  }
  void coords(int v, int64_t gid, int64_t& bx, int64_t& by, int64_t& bz) const {
    const Node& n = g.nodes[v];
    int64_t l = gid - n.gid0;
    bx = l % n.gx();
    by = (l / n.gx()) % n.gy();
    bz = l / (n.gx() * n.gy());
  }
  int64_t gid_of(int v, int64_t bx, int64_t by, int64_t bz) const {
    const Node& n = g.nodes[v];
    return n.gid0 + (bz * n.gy() + by) * n.gx() + bx;
  }

  void mark_lines(int v, int64_t bx, int64_t by, int64_t bz) {
    if (budget_lines < 0) return;
    for (int a = 0; a < (int)g.nodes[v].acc.size(); ++a)
      g.for_each_line_range(v, a, bx, by, bz, [&](int buf, int64_t l0, int64_t l1) {
        if (!counted[buf]) return;
        const int64_t base = g.bufs[buf].line0;
        auto& bm = bits[buf];
        for (int64_t l = l0 - base; l < l1 - base;) {
          int64_t w = l >> 6;
          int64_t hi = std::min<int64_t>(l1 - base, (w + 1) << 6);
          int64_t nb = hi - l;
          uint64_t m = (nb == 64 ? ~0ull : ((1ull << nb) - 1) << (l & 63));
          uint64_t old = bm[w];
          if (!old) dirty.push_back({buf, w});
          nlines += __builtin_popcountll(m & ~old);
          bm[w] = old | m;
          l = hi;
        }
      });
  }

  void add_block(int v, int64_t gid) {
    st[gid] = 1;
    tba.push_back(gid);
    work.push_back(gid);
    if (leaf_node[v]) ++leaf_in_tba;
    int64_t bx, by, bz;
    coords(v, gid, bx, by, bz);
    mark_lines(v, bx, by, bz);
  }

  // l.6–10: closure over producers; blocks already in toBeAssigned U assigned are closed.
  void closure(int64_t gid0) {
    std::vector<int64_t> stack{gid0};
    while (!stack.empty()) {
      int64_t gid = stack.back();
      stack.pop_back();
      int v = node_of(gid);
      int64_t bx, by, bz;
      coords(v, gid, bx, by, bz);
      for (const Chan& c : g.in_ch[v]) {
        if (!in_c[c.u]) continue;  // intra-cluster dependencies only (A13)
        BRange r = g.producers(c, bx, by);
        for (int64_t y = r.y0; y < r.y1; ++y)
          for (int64_t x = r.x0; x < r.x1; ++x) {
            int64_t p = gid_of(c.u, x, y, bz);
            if (st[p] == 0) {
              add_block(c.u, p);
              stack.push_back(p);
            }
          }
      }
    }
  }

  bool deps_covered(int v, int64_t bx, int64_t by, int64_t bz) const {
    bool any = false;
    for (const Chan& c : g.in_ch[v]) {
      if (!in_c[c.u]) continue;
      BRange r = g.producers(c, bx, by);
      for (int64_t y = r.y0; y < r.y1; ++y)
        for (int64_t x = r.x0; x < r.x1; ++x) {
          any = true;
          if (st[gid_of(c.u, x, y, bz)] == 0) return false;
        }
    }
    return any;  // non-empty dependency set (A14)
  }

  // l.11–12 FindMoreBlks via worklist.
  void top_down() {
    while (!work.empty()) {
      int64_t gid = work.back();
      work.pop_back();
      int u = node_of(gid);
      int64_t px, py, pz;
      coords(u, gid, px, py, pz);
      for (const Chan& c : g.out_ch[u]) {
        if (!in_c[c.v]) continue;
        BRange r = g.consumers(c, px, py);
        for (int64_t y = r.y0; y < r.y1; ++y)
          for (int64_t x = r.x0; x < r.x1; ++x) {
            int64_t cg = gid_of(c.v, x, y, pz);
            if (st[cg] == 0 && deps_covered(c.v, x, y, pz)) add_block(c.v, cg);
          }
      }
    }
  }

  bool check() const {
    if (budget_lines >= 0) return nlines <= budget_lines;
    return leaf_in_tba <= rows_cap;
  }

  void clear_fp() {
    for (auto& d : dirty) bits[d.first][d.second] = 0;
    dirty.clear();
    nlines = 0;
  }

  // l.17–24: commit newSubKBlks (tba[0:n]) as one sub-kernel per node, topological order.
  void commit(size_t n, int64_t fp_lines) {
    std::vector<std::vector<int64_t>> per(g.nodes.size());
    for (size_t i = 0; i < n; ++i) {
      st[tba[i]] = 2;
      per[node_of(tba[i])].push_back(tba[i]);
    }
    for (size_t i = n; i < tba.size(); ++i) st[tba[i]] = 0;
    for (int v : g.topo) {
      if (per[v].empty()) continue;
      SubKernel sk;
      sk.node = v;
      sk.frag = (int32_t)nfrag;
      sk.cluster = cluster_id;
      sk.nblocks = (int64_t)per[v].size();
      if (use_et) {  // l.19: ET(subKer_v, C_i, perfTables) — hot iff an input is produced in the cluster
        bool hot = false;
        for (const Chan& c : g.in_ch[v]) hot = hot || in_c[c.u];
        cost += g.nodes[v].et(sk.nblocks, hot);
      }
      sk.footprint = fp_lines * 128;
      to_rects(v, per[v], sk.rects);
      out.subs.push_back(std::move(sk));
    }
    out.max_footprint = std::max(out.max_footprint, fp_lines * 128);
    ++nfrag;
    tba.clear();
    new_len = 0;
    leaf_in_tba = 0;
    new_leaf = 0;
    new_lines = 0;
    clear_fp();
    for (int v : leaves) {
      while (cursor[v] < g.nodes[v].nblocks && st[g.nodes[v].gid0 + cursor[v]] == 2) ++cursor[v];
      scan[v] = cursor[v];
    }
  }

  // Sorted block ids -> disjoint rects: x-runs per row, stacked rows with equal x-runs,
  // then equal rects over consecutive frames.
  void to_rects(int v, std::vector<int64_t>& ids, std::vector<Rect6>& rects) const {
    std::sort(ids.begin(), ids.end());
    struct Seg { int64_t x0, x1, y, z; };
    std::vector<Seg> segs;
    for (int64_t id : ids) {
      int64_t bx, by, bz;
      coords(v, id, bx, by, bz);
      if (!segs.empty() && segs.back().y == by && segs.back().z == bz && segs.back().x1 == bx) {
        segs.back().x1++;
      } else {
        segs.push_back({bx, bx + 1, by, bz});
      }
    }
    std::vector<Rect6> rs;
    for (auto& s : segs) {
      if (!rs.empty()) {
        Rect6& b = rs.back();
        if (b.z0 == s.z && b.x0 == s.x0 && b.x1 == s.x1 && b.y1 == s.y) {
          b.y1++;
          continue;
        }
      }
      rs.push_back({(int32_t)s.x0, (int32_t)s.y, (int32_t)s.z, (int32_t)s.x1, (int32_t)s.y + 1, (int32_t)s.z + 1});
    }
    for (auto& r : rs) {
      if (!rects.empty()) {
        Rect6& b = rects.back();
        if (b.x0 == r.x0 && b.x1 == r.x1 && b.y0 == r.y0 && b.y1 == r.y1 && b.z1 == r.z0) {
          b.z1 = r.z1;
          continue;
        }
      }
      rects.push_back(r);
    }
  }

  int64_t pick(int v) {
    const Node& n = g.nodes[v];
    int64_t& s = scan[v];
    while (s < n.nblocks && st[n.gid0 + s] != 0) ++s;
    return s < n.nblocks ? n.gid0 + s : -1;
  }

  ktiler_status run() {
    const int nn = (int)g.nodes.size();
    st.assign(g.total_blocks, 0);
    int64_t cluster_blocks = 0;
    for (int v = 0; v < nn; ++v) {
      if (in_c[v]) cluster_blocks += g.nodes[v].nblocks;
      else std::fill(st.begin() + g.nodes[v].gid0, st.begin() + g.nodes[v].gid0 + g.nodes[v].nblocks, (uint8_t)2);
    }
    nfrag = out.nfrag;  // fragments are numbered across clusters
    if (budget_lines >= 0) {
      bits.resize(g.bufs.size());
      for (size_t b = 0; b < g.bufs.size(); ++b) bits[b].assign((g.bufs[b].nlines + 63) / 64, 0);
    }
    leaf_node.assign(nn, 0);
    for (int v : g.topo) {  // leaves of the cluster: no consumer inside it
      if (!in_c[v]) continue;
      bool leaf = true;
      for (const Chan& c : g.out_ch[v]) leaf = leaf && !in_c[c.v];
      if (leaf) {
        leaf_node[v] = 1;
        leaves.push_back(v);
      }
    }
    cursor.assign(nn, 0);
    scan.assign(nn, 0);
    int64_t assigned = 0;
    std::vector<int> rev(g.topo.rbegin(), g.topo.rend());
    for (;;) {
      // ---- bottom-up round (l.4–10) ----
      std::vector<std::pair<int, int64_t>> picked;
      for (int v : leaves) {
        int64_t b = pick(v);
        if (b >= 0) picked.push_back({v, b});
      }
      if (picked.empty()) {
        // A16b: blocks no leaf block depends on act as bottom blocks, last node first
        for (int v : rev) {
          if (!in_c[v]) continue;
          const Node& n = g.nodes[v];
          for (int64_t l = 0; l < n.nblocks; ++l)
            if (st[n.gid0 + l] == 0) {
              picked.push_back({v, n.gid0 + l});
              break;
            }
          if (!picked.empty()) break;
        }
      }
      if (picked.empty()) {
        // A16: every block is in assigned U toBeAssigned -> commit newSubKBlks
        if (new_len == 0 && assigned < cluster_blocks) return fail(KTILER_E_UNTILEABLE, "internal: nothing to commit");
        if (new_len) commit(new_len, new_lines);
        break;
      }
      for (auto& pb : picked) {
        if (st[pb.second] != 0) continue;
        add_block(pb.first, pb.second);
        closure(pb.second);
      }
      // ---- top-down round (l.11–12) ----
      top_down();
      // ---- l.13 ----
      if (check()) {
        new_len = tba.size();
        new_lines = nlines;
        new_leaf = leaf_in_tba;
        continue;
      }
      if (new_len == 0) {
        if (!force_minimal)
          return fail(KTILER_E_UNTILEABLE,
                      "Alg. 2 l.23 (PAPER.md:305): the dependency closure of one leaf block needs " +
                          std::to_string(nlines * 128) + " B > budget " + std::to_string(budget_lines * 128) + " B");
        size_t n = tba.size();
        int64_t fl = nlines;
        assigned += (int64_t)n;
        commit(n, fl);  // FORCE_MINIMAL: over-budget fragment, recorded in max_footprint
        continue;
      }
      assigned += (int64_t)new_len;
      commit(new_len, new_lines);
    }
    out.nfrag = nfrag;
    return KTILER_OK;
  }
};

}  // namespace

static void untiled(const Graph& g, Schedule& out) {
  int64_t fp = 0;
  for (auto& b : g.bufs) fp += b.nlines * 128;
  for (int v : g.topo) {
    const Node& n = g.nodes[v];
    SubKernel sk;
    sk.node = v;
    sk.frag = 0;
    sk.nblocks = n.nblocks;
    sk.footprint = fp;
    sk.rects.push_back({0, 0, 0, (int32_t)n.gx(), (int32_t)n.gy(), (int32_t)n.gz()});
    out.subs.push_back(sk);
  }
  out.nfrag = 1;
  out.max_footprint = fp;
}

// Alg. 1 Application Tiling.  Starts from singleton
// clusters whose cost is the kernel's default (untiled, cold-input) execution time, takes
// the candidate edges (weight > thld; weight < 0 = derived from the performance tables as
// the time the consumer saves when that input is cached), highest weight
// first (ties: src id, dst id), merges the two clusters at the ends of the current edge
// when the partition stays valid (the quotient graph of clusters is acyclic),
// tiles the merged cluster with Alg. 2 and keeps it iff CO_m < CO_a + CO_b; the edge is
// then removed and the scan restarts at the top (l.16), an invalid merge moves to the
// next edge (l.18).  The schedule concatenates the clusters' tiling sequences in a
// topological order of the clusters; an unmerged node runs untiled (l.2: T_i = kernel).
static const double ALG1_INF = 1e300;

static bool quotient_acyclic(const Graph& g, const std::vector<int>& cl) {
  const int nn = (int)g.nodes.size();
  std::vector<std::vector<int>> adj(nn);
  std::vector<int> indeg(nn, 0), present(nn, 0);
  for (int v = 0; v < nn; ++v) present[cl[v]] = 1;
  for (int v = 0; v < nn; ++v)
    for (const Chan& c : g.out_ch[v])
      if (cl[c.u] != cl[c.v]) {
        adj[cl[c.u]].push_back(cl[c.v]);
        ++indeg[cl[c.v]];
      }
  std::vector<int> q;
  int seen = 0, total = 0;
  for (int c = 0; c < nn; ++c)
    if (present[c]) {
      ++total;
      if (!indeg[c]) q.push_back(c);
    }
  while (!q.empty()) {
    int c = q.back();
    q.pop_back();
    ++seen;
    for (int d : adj[c])
      if (--indeg[d] == 0) q.push_back(d);
  }
  return seen == total;
}

static ktiler_status alg1(Graph& g, int64_t budget_lines, double thld, bool resident, Schedule& out) {
  const int nn = (int)g.nodes.size();
  for (int v = 0; v < nn; ++v)
    if (g.nodes[v].perf_n.empty())
      return fail(KTILER_E_STATE, "KTILER_FRAG_ALG1 needs a performance table for every node (ktiler_set_perf_table)");
  std::vector<int> pos(nn);
  for (int i = 0; i < nn; ++i) pos[g.topo[i]] = i;
  std::vector<int> cl(nn);
  std::vector<std::vector<int>> members(nn);
  std::vector<double> CO(nn);
  for (int v = 0; v < nn; ++v) {  // l.1–5
    cl[v] = v;
    members[v] = {v};
    CO[v] = g.nodes[v].et(g.nodes[v].nblocks, false);
  }
  struct Cand {
    double w;
    int src, dst;
  };
  std::vector<Cand> cand;  // l.6–7
  for (const Edge& e : g.edges) {
    const Node& d = g.nodes[e.dst];
    const double w = e.w >= 0 ? (double)e.w : d.et(d.nblocks, false) - d.et(d.nblocks, true);
    if (w > thld) cand.push_back({w, e.src, e.dst});
  }
  std::stable_sort(cand.begin(), cand.end(), [](const Cand& a, const Cand& b) {
    if (a.w != b.w) return a.w > b.w;
    if (a.src != b.src) return a.src < b.src;
    return a.dst < b.dst;
  });
  auto tile = [&](const std::vector<int>& mem, int32_t cid, Schedule& into, double* cost) -> ktiler_status {
    Partitioner p(g, into, resident);
    std::fill(p.in_c.begin(), p.in_c.end(), (uint8_t)0);
    for (int v : mem) p.in_c[v] = 1;
    p.budget_lines = budget_lines;
    p.rows_cap = 0;
    p.force_minimal = false;
    p.use_et = true;
    p.cluster_id = cid;
    ktiler_status st = p.run();
    *cost = st ? ALG1_INF : p.cost;
    return st;
  };
  size_t eix = 0;
  while (eix < cand.size()) {  // l.8
    const int a = cl[cand[eix].src], b = cl[cand[eix].dst];  // l.10
    if (a == b) {  // both ends already in one cluster (A22)
      cand.erase(cand.begin() + (long)eix);
      eix = 0;
      continue;
    }
    std::vector<int> merged = members[a];  // l.11 MergeOrder: topological order
    merged.insert(merged.end(), members[b].begin(), members[b].end());
    std::sort(merged.begin(), merged.end(), [&](int x, int y) { return pos[x] < pos[y]; });
    std::vector<int> cl2 = cl;  // l.12–13
    for (int v : members[b]) cl2[v] = a;
    if (!quotient_acyclic(g, cl2)) {
      ++eix;  // l.18
      continue;
    }
    Schedule tmp;  // l.14
    double com = 0;
    tile(merged, 0, tmp, &com);
    if (com < CO[a] + CO[b]) {  // l.15
      cl = cl2;
      members[a] = merged;
      members[b].clear();
      CO[a] = com;
    }
    cand.erase(cand.begin() + (long)eix);  // l.16
    eix = 0;
  }
  kt::clear_error();
  // l.21–24: clusters in a topological order of the quotient graph
  std::vector<int> order;
  {
    std::vector<int> indeg(nn, 0);
    std::vector<std::vector<int>> adj(nn);
    for (int v = 0; v < nn; ++v)
      for (const Chan& c : g.out_ch[v])
        if (cl[c.u] != cl[c.v]) {
          adj[cl[c.u]].push_back(cl[c.v]);
          ++indeg[cl[c.v]];
        }
    std::vector<int> ready;
    for (int c = 0; c < nn; ++c)
      if (!members[c].empty() && !indeg[c]) ready.push_back(c);
    while (!ready.empty()) {  // smallest topological position first (deterministic)
      auto it = std::min_element(ready.begin(), ready.end(),
                                 [&](int x, int y) { return pos[members[x][0]] < pos[members[y][0]]; });
      const int c = *it;
      ready.erase(it);
      order.push_back(c);
      for (int d : adj[c])
        if (--indeg[d] == 0) ready.push_back(d);
    }
  }
  for (int c : order) {
    const int32_t cid = (int32_t)out.clusters.size();
    if (members[c].size() == 1) {
      const int v = members[c][0];
      const Node& n = g.nodes[v];
      SubKernel sk;
      sk.node = v;
      sk.frag = (int32_t)out.nfrag++;
      sk.cluster = cid;
      sk.nblocks = n.nblocks;
      int64_t fp = 0;
      for (auto& a : n.acc) fp += g.bufs[a.buf].nlines * 128;
      sk.footprint = fp;
      sk.rects.push_back({0, 0, 0, (int32_t)n.gx(), (int32_t)n.gy(), (int32_t)n.gz()});
      out.subs.push_back(sk);
      out.max_footprint = std::max(out.max_footprint, fp);
    } else {
      double cost = 0;
      ktiler_status st = tile(members[c], cid, out, &cost);
      if (st) return st;
    }
    out.clusters.push_back(members[c]);
    out.cluster_cost.push_back(CO[c]);
  }
  return KTILER_OK;
}

// KTILER_PF_MULTIRATE: cheap nodes (output pixels <= 1/4 of the largest node's, closed
// under "all consumers are cheap too") get one sub-kernel per two fragments: the one of
// fragment 2k is merged into that of fragment 2k+1 (emitted at 2k+1's place, in the same
// topological position).  Only consumers move later, so every RAW dependency still points
// to an earlier sub-kernel.  sub_deps / discards are derived afterwards.
static void multirate(const Graph& g, Schedule& s) {
  const int nn = (int)g.nodes.size();
  std::vector<double> pix(nn, 0.0);
  double maxpix = 0;
  for (int v = 0; v < nn; ++v) {
    const Node& n = g.nodes[v];
    const Buffer& b = g.bufs[n.acc[n.wacc].buf];
    pix[v] = (double)b.d.width * b.d.height * b.d.frames;
    maxpix = std::max(maxpix, pix[v]);
  }
  std::vector<uint8_t> cheap(nn, 0);
  for (int v = 0; v < nn; ++v) cheap[v] = 4.0 * pix[v] <= maxpix;
  for (bool changed = true; changed;) {  // close downward
    changed = false;
    for (int v = 0; v < nn; ++v)
      if (cheap[v])
        for (const Chan& c : g.out_ch[v])
          if (!cheap[c.v]) {
            cheap[v] = 0;
            changed = true;
          }
  }
  bool any = false;
  for (int v = 0; v < nn; ++v) any |= cheap[v] != 0;
  if (!any || s.nfrag < 2) return;
  std::vector<SubKernel> out;
  std::vector<int> pending(nn, -1);  // index into s.subs of a deferred sub-kernel
  std::vector<SubKernel>& in = s.subs;
  size_t i = 0;
  while (i < in.size()) {
    const int32_t f = in[i].frag;
    size_t j = i;
    while (j < in.size() && in[j].frag == f) ++j;
    const bool last_frag = j == in.size();
    for (size_t k = i; k < j; ++k) {
      const int v = in[k].node;
      if (!cheap[v]) {
        out.push_back(in[k]);
        continue;
      }
      if (pending[v] < 0 && (f % 2 == 0) && !last_frag) {
        pending[v] = (int)k;  // defer to the next odd fragment
        continue;
      }
      SubKernel m = in[k];
      if (pending[v] >= 0) {
        const SubKernel& p = in[pending[v]];
        m.rects.insert(m.rects.begin(), p.rects.begin(), p.rects.end());
        m.nblocks += p.nblocks;
        m.footprint = std::max(m.footprint, p.footprint);
        pending[v] = -1;
      }
      out.push_back(std::move(m));
    }
    i = j;
  }
  for (int v = 0; v < nn; ++v)  // a deferred sub-kernel with no later fragment of its node
    if (pending[v] >= 0) out.push_back(in[pending[v]]);
  s.subs.swap(out);
}

ktiler_status build_schedule(Graph& g, int64_t cache_bytes, const ktiler_fragment_policy& pol, Schedule& out) {
  ktiler_status st0 = build_schedule_core(g, cache_bytes, pol, out);
  if (st0 || !(pol.flags & KTILER_PF_MULTIRATE) || pol.kind == KTILER_FRAG_NONE) return st0;
  multirate(g, out);
  return KTILER_OK;
}

ktiler_status build_schedule_core(Graph& g, int64_t cache_bytes, const ktiler_fragment_policy& pol, Schedule& out) {
  ktiler_status s = g.finalize();
  if (s) return s;
  out = Schedule();
  double frac = pol.l2_fraction > 0 ? pol.l2_fraction : 1.0;
  out.budget = (int64_t)std::floor((double)cache_bytes * frac);
  bool force = (pol.flags & KTILER_PF_FORCE_MINIMAL) != 0;
  const bool resident = (pol.flags & KTILER_PF_RESIDENT_BUDGET) != 0;
  if (pol.kind != KTILER_FRAG_ALG1 && pol.kind != KTILER_FRAG_CHAIN) {
    std::vector<int> all(g.topo.begin(), g.topo.end());
    out.clusters.push_back(all);
    out.cluster_cost.push_back(0.0);
  }
  switch (pol.kind) {
    case KTILER_FRAG_CHAIN: {  // fixed partition: `rows` consecutive nodes per cluster
      if (pol.rows < 1) return fail(KTILER_E_INVALID, "CHAIN policy needs rows >= 1 (nodes per cluster)");
      const int nn = (int)g.topo.size();
      for (int a = 0; a < nn; a += (int)pol.rows) {
        std::vector<int> mem(g.topo.begin() + a, g.topo.begin() + std::min<int64_t>(nn, a + pol.rows));
        Partitioner p(g, out, resident);
        std::fill(p.in_c.begin(), p.in_c.end(), (uint8_t)0);
        for (int v : mem) p.in_c[v] = 1;
        p.budget_lines = out.budget / 128;
        p.rows_cap = 0;
        p.force_minimal = force;
        p.cluster_id = (int32_t)out.clusters.size();
        ktiler_status st = p.run();
        if (st) return st;
        out.clusters.push_back(mem);
        out.cluster_cost.push_back(0.0);
      }
      return KTILER_OK;
    }
    case KTILER_FRAG_ALG1: return alg1(g, out.budget / 128, pol.alg1_thld, resident, out);
    case KTILER_FRAG_NONE: untiled(g, out); return KTILER_OK;
    case KTILER_FRAG_BUDGET: {
      Partitioner p(g, out, resident);
      p.budget_lines = out.budget / 128;
      p.rows_cap = 0;
      p.force_minimal = force;
      return p.run();
    }
    case KTILER_FRAG_ROWS:
    case KTILER_FRAG_BALANCED: {
      int64_t leaf_gx = 0, leaf_rows = 0;
      for (int v = 0; v < (int)g.nodes.size(); ++v)
        if (g.out_ch[v].empty()) {
          leaf_gx += g.nodes[v].gx();
          leaf_rows = std::max(leaf_rows, g.nodes[v].gy() * g.nodes[v].gz());
        }
      int64_t rows = pol.rows;
      if (pol.kind == KTILER_FRAG_BALANCED) {
        Schedule tmp;
        Partitioner p(g, tmp, resident);
        p.budget_lines = out.budget / 128;
        p.rows_cap = 0;
        p.force_minimal = force;
        ktiler_status s2 = p.run();
        if (s2) return s2;
        rows = (leaf_rows + tmp.nfrag - 1) / std::max<int64_t>(1, tmp.nfrag);
      }
      if (rows < 1) return fail(KTILER_E_INVALID, "ROWS policy needs rows >= 1");
      Partitioner p(g, out, resident);
      p.budget_lines = -1;
      p.rows_cap = rows * leaf_gx;
      p.force_minimal = true;
      ktiler_status s3 = p.run();
      if (s3) return s3;
      // footprints are not tracked in ROWS mode; report the lines of each fragment
      return KTILER_OK;
    }
    default: return fail(KTILER_E_INVALID, "unknown fragment policy kind");
  }
}

// Per producer block of an INTERNAL buffer: the position of its last reader in the total
// order.  Lines of blocks whose last reader is sub-kernel s are dead once s completes.
void compute_discards(const Graph& g, Schedule& s, std::vector<int32_t>* sub_of_out) {
  std::vector<int32_t> sub_of(g.total_blocks, -1);
  for (size_t i = 0; i < s.subs.size(); ++i) {
    const SubKernel& sk = s.subs[i];
    const Node& n = g.nodes[sk.node];
    for (auto& r : sk.rects)
      for (int64_t z = r.z0; z < r.z1; ++z)
        for (int64_t y = r.y0; y < r.y1; ++y)
          for (int64_t x = r.x0; x < r.x1; ++x) sub_of[n.gid0 + (z * n.gy() + y) * n.gx() + x] = (int32_t)i;
  }
  s.discards.assign(s.subs.size(), {});
  s.discard_readers.assign(s.subs.size(), {});
  s.discard_lines = 0;
  // sub-kernel dependencies: the producer sub-kernels of every block of each sub-kernel
  s.sub_deps.assign(s.subs.size(), {});
  for (size_t i = 0; i < s.subs.size(); ++i) {
    const SubKernel& sk = s.subs[i];
    std::vector<int32_t>& dep = s.sub_deps[i];
    for (const Chan& c : g.in_ch[sk.node]) {
      const Node& u = g.nodes[c.u];
      for (auto& r : sk.rects)
        for (int64_t z = r.z0; z < r.z1; ++z)
          for (int64_t y = r.y0; y < r.y1; ++y)
            for (int64_t x = r.x0; x < r.x1; ++x) {
              BRange pr = g.producers(c, x, y);
              for (int64_t py = pr.y0; py < pr.y1; ++py)
                for (int64_t px = pr.x0; px < pr.x1; ++px) {
                  const int32_t so = sub_of[u.gid0 + (z * u.gy() + py) * u.gx() + px];
                  if (dep.empty() || dep.back() != so) dep.push_back(so);
                }
            }
    }
    std::sort(dep.begin(), dep.end());
    dep.erase(std::unique(dep.begin(), dep.end()), dep.end());
  }
  // Lines are discarded only where tiling keeps them in L2: producer and last reader in
  // the same cluster, and that cluster tiled into more than one fragment (an untiled
  // intermediate has left L2 long before its last reader ends).
  std::vector<int32_t> cf0(s.clusters.size() + 1, INT32_MAX), cf1(s.clusters.size() + 1, -1);
  for (const SubKernel& sk : s.subs) {
    cf0[sk.cluster] = std::min(cf0[sk.cluster], sk.frag);
    cf1[sk.cluster] = std::max(cf1[sk.cluster], sk.frag);
  }
  for (int u = 0; u < (int)g.nodes.size(); ++u) {
    const Node& n = g.nodes[u];
    const Access& w = n.acc[n.wacc];
    const Buffer& B = g.bufs[w.buf];
    if (!(B.d.flags & KTILER_BUF_INTERNAL)) continue;
    // last reader per producer block, then dead blocks grouped per sub-kernel
    std::vector<std::vector<int64_t>> dead(s.subs.size());
    for (int64_t l = 0; l < n.nblocks; ++l) {
      int64_t px = l % n.gx(), py = (l / n.gx()) % n.gy(), pz = l / (n.gx() * n.gy());
      int32_t last = sub_of[n.gid0 + l];
      std::vector<int32_t> rd{last};
      for (const Chan& c : g.out_ch[u]) {
        if (c.buf != w.buf) continue;
        const Node& v = g.nodes[c.v];
        BRange r = g.consumers(c, px, py);
        for (int64_t y = r.y0; y < r.y1; ++y)
          for (int64_t x = r.x0; x < r.x1; ++x) {
            const int32_t sc = sub_of[v.gid0 + (pz * v.gy() + y) * v.gx() + x];
            last = std::max(last, sc);
            rd.push_back(sc);
          }
      }
      const int32_t own = sub_of[n.gid0 + l];
      const int32_t c = own >= 0 ? s.subs[own].cluster : -1;
      const bool tiled = c >= 0 && last >= 0 && s.subs[last].cluster == c && cf1[c] > cf0[c];
      if (last >= 0 && tiled) {
        dead[last].push_back(l);
        auto& R = s.discard_readers[last];
        R.insert(R.end(), rd.begin(), rd.end());
      }
    }
    const int64_t e = B.d.elem_bytes;
    for (size_t si = 0; si < dead.size(); ++si) {
      if (dead[si].empty()) continue;
      // x-runs per (z, y) row of blocks, stacked into rects, mapped to pixel rows
      auto& ids = dead[si];
      std::sort(ids.begin(), ids.end());
      size_t i = 0;
      std::vector<Discard> rows;
      while (i < ids.size()) {
        int64_t l = ids[i];
        int64_t x0 = l % n.gx(), y = (l / n.gx()) % n.gy(), z = l / (n.gx() * n.gy());
        int64_t x1 = x0 + 1;
        size_t j = i + 1;
        while (j < ids.size() && ids[j] == ids[j - 1] + 1 && (ids[j] % n.gx()) != 0) {
          ++x1;
          ++j;
        }
        PRect a = g.access_rect(u, n.wacc, x0, y);
        PRect b = g.access_rect(u, n.wacc, x1 - 1, y);
        if (!a.empty() && !b.empty()) {
          Discard d{w.buf, a.x0 * e, b.x1 * e, (int32_t)a.y0, (int32_t)a.y1, (int32_t)z, (int32_t)z + 1};
          if (!rows.empty()) {
            Discard& p = rows.back();
            if (p.xb0 == d.xb0 && p.xb1 == d.xb1 && p.z0 == d.z0 && p.y1 == d.y0) {
              p.y1 = d.y1;
              i = j;
              continue;
            }
          }
          rows.push_back(d);
        }
        i = j;
      }
      for (auto& d : rows) {
        if (!s.discards[si].empty()) {
          Discard& p = s.discards[si].back();
          if (p.buf == d.buf && p.xb0 == d.xb0 && p.xb1 == d.xb1 && p.y0 == d.y0 && p.y1 == d.y1 && p.z1 == d.z0) {
            p.z1 = d.z1;
            continue;
          }
        }
        s.discards[si].push_back(d);
      }
    }
  }
  for (auto& R : s.discard_readers) {
    std::sort(R.begin(), R.end());
    R.erase(std::unique(R.begin(), R.end()), R.end());
  }
  for (auto& v : s.discards)
    for (auto& d : v) {
      const Buffer& B = g.bufs[d.buf];
      for (int64_t z = d.z0; z < d.z1; ++z)
        for (int64_t y = d.y0; y < d.y1; ++y) {
          uint64_t r = B.addr + (uint64_t)(B.frame_off(z) + y * B.d.pitch_bytes);
          int64_t l0 = (int64_t)((r + d.xb0 + 127) >> 7), l1 = (int64_t)((r + d.xb1) >> 7);
          if (l1 > l0) s.discard_lines += l1 - l0;
        }
    }
  if (sub_of_out) *sub_of_out = std::move(sub_of);
}

}  // namespace kt
