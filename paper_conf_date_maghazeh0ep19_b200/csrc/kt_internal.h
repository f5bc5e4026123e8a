// Internal structures of libktiler (host side).  Not part of the ABI.
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "ktiler.h"

namespace kt {

// ---- error reporting (thread-local message behind ktiler_last_error) ----
void set_error(const std::string& msg);
void clear_error();
ktiler_status fail(ktiler_status s, const std::string& msg);

inline int64_t floordiv(int64_t a, int64_t b) {  // b > 0
  int64_t q = a / b;
  return (a % b != 0 && a < 0) ? q - 1 : q;
}

struct Buffer {
  ktiler_buffer_desc d;
  // byte offset of frame z (a ring buffer keeps frame z in slot z mod ring_frames)
  int64_t frame_off(int64_t z) const { return (d.ring_frames ? z % d.ring_frames : z) * d.frame_stride_bytes; }
  int64_t span = 0;   // bytes from base to the end of the last frame's last row
  uint64_t addr = 0;  // (uint64_t)base
  int64_t line0 = 0;  // addr >> 7
  int64_t nlines = 0; // lines spanned
  int writer = -1;    // node writing it (at most one)
  std::vector<int> readers;
};

struct Access {
  int32_t buf = -1, mode = 0;
  int64_t ax = 1, ay = 1, ox = 0, oy = 0;
  int32_t hl = 0, hr = 0, ht = 0, hb = 0;
};

struct Node {
  int32_t op = 0;
  uint32_t grid[3] = {1, 1, 1}, block[3] = {1, 1, 1};
  std::vector<Access> acc;
  std::vector<uint8_t> params;
  ktiler_launch_fn launch = nullptr;
  void* user = nullptr;
  int wacc = -1;     // index of the (single) WRITE access for built-ins
  int racc = -1;     // index of the (first) READ access for built-ins
  int racc2 = -1;    // KTILER_OP_JACOBI: its second READ access (the coefficients)
  int radius = 0;    // KTILER_OP_GAUSS_F32: ceil(3 sigma)
  float taps[9] = {};  // KTILER_OP_GAUSS_F32: f64-normalised Gaussian weights rounded to f32
  int64_t nblocks = 0;
  int64_t gid0 = 0;  // first global block id
  float T = 200.f;
  bool scalar = false;  // one thread per pixel variant
  // performance table: execution time (ms) of a sub-kernel of perf_n[k]
  // blocks with its input cold (HBM) / hot (produced by tiling, in L2); empty = none
  std::vector<int64_t> perf_n;
  std::vector<double> perf_cold, perf_hot;
  // ET lookup (A35): piecewise linear in the block count, the first point's time below
  // the table, the last point's per-block rate above it
  double et(int64_t n, bool hot) const {
    const std::vector<double>& t = hot ? perf_hot : perf_cold;
    const size_t m = perf_n.size();
    if (m == 0) return (double)n;
    if (n <= perf_n[0]) return t[0];
    for (size_t k = 1; k < m; ++k)
      if (n <= perf_n[k])
        return t[k - 1] + (t[k] - t[k - 1]) * (double)(n - perf_n[k - 1]) / (double)(perf_n[k] - perf_n[k - 1]);
    return t[m - 1] * (double)n / (double)perf_n[m - 1];
  }
  int64_t gx() const { return grid[0]; }
  int64_t gy() const { return grid[1]; }
  int64_t gz() const { return grid[2]; }
  int64_t nthreads() const { return (int64_t)block[0] * block[1] * block[2]; }
};

struct Edge {
  int32_t src, dst, buf;
  float w;
};

// Half-open pixel rectangle in one frame (clipped to a buffer).
struct PRect {
  int64_t x0, y0, x1, y1;
  bool empty() const { return x0 >= x1 || y0 >= y1; }
};

// Half-open block range.
struct BRange {
  int64_t x0, x1, y0, y1;
  bool empty() const { return x0 >= x1 || y0 >= y1; }
};

// One dependency "channel": consumer node v reads buffer X (access r) written by node u
// (access w).  Both directions are closed forms of the affine maps.
struct Chan {
  int v, r, u, w, buf;
};

struct Graph {
  std::vector<Buffer> bufs;
  std::vector<Node> nodes;
  std::vector<Edge> edges;
  // derived by finalize()
  std::vector<int> topo;                 // topological order of nodes
  std::vector<std::vector<Chan>> in_ch;  // per consumer node
  std::vector<std::vector<Chan>> out_ch; // per producer node
  int64_t total_blocks = 0;
  bool finalized = false;

  // Does any node write buffer b?  (false: a graph input)
  bool written_by_node(int b) const {
    for (auto& n : nodes)
      for (auto& a : n.acc)
        if (a.buf == b && a.mode == KTILER_WRITE) return true;
    return false;
  }

  ktiler_status finalize();  // validate + derive; idempotent

  PRect access_rect(int node, int acc, int64_t bx, int64_t by) const;
  // producer blocks of node c.u touched by consumer block (bx, by) through channel c
  BRange producers(const Chan& c, int64_t bx, int64_t by) const;
  // consumer blocks of node c.v whose reads touch producer block (px, py) through channel c
  BRange consumers(const Chan& c, int64_t px, int64_t py) const;
  // line ranges [l0, l1) (absolute line ids) touched by one access of one block
  template <class F>
  void for_each_line_range(int node, int acc, int64_t bx, int64_t by, int64_t bz, F&& f) const;
};

template <class F>
void Graph::for_each_line_range(int node, int acc, int64_t bx, int64_t by, int64_t bz, F&& f) const {
  const Node& n = nodes[node];
  const Access& a = n.acc[acc];
  const Buffer& b = bufs[a.buf];
  PRect r = access_rect(node, acc, bx, by);
  if (r.empty()) return;
  const int64_t e = b.d.elem_bytes;
  const uint64_t fb = b.addr + (uint64_t)b.frame_off(bz);
  for (int64_t y = r.y0; y < r.y1; ++y) {
    uint64_t lo = fb + (uint64_t)(y * b.d.pitch_bytes + r.x0 * e);
    uint64_t hi = fb + (uint64_t)(y * b.d.pitch_bytes + r.x1 * e);  // exclusive
    f(a.buf, (int64_t)(lo >> 7), (int64_t)((hi - 1) >> 7) + 1);
  }
}

// ---- plan ----
struct Rect6 {
  int32_t x0, y0, z0, x1, y1, z1;
  int64_t count() const { return (int64_t)(x1 - x0) * (y1 - y0) * (z1 - z0); }
};

struct SubKernel {
  int32_t node = 0, frag = 0;
  int32_t cluster = 0;    // Alg. 1 cluster (0 when the whole graph is one cluster)
  int64_t nblocks = 0;
  int64_t footprint = 0;  // bytes, of the fragment
  std::vector<Rect6> rects;
};

// Lines of one buffer to discard: rows [y0,y1) of frames [z0,z1), byte columns [xb0,xb1)
// (128-B aligned absolute line boundaries are applied at launch).
struct Discard {
  int32_t buf;
  int64_t xb0, xb1;
  int32_t y0, y1, z0, z1;
};

struct Schedule {
  std::vector<SubKernel> subs;  // total order ("a total order")
  int64_t nfrag = 0;
  int64_t budget = 0;
  int64_t max_footprint = 0;
  // discards[i] = ranges that become dead once subs[i] has completed
  std::vector<std::vector<Discard>> discards;
  int64_t discard_lines = 0;
  // sub-kernel dependency sets (a sub-kernel depends on another iff one
  // of its blocks depends on one of the other's) and, per discard list, every sub-kernel
  // that reads the dying blocks (a discard may only run after all of them) — GRAPH_DAG
  std::vector<std::vector<int32_t>> sub_deps;
  std::vector<std::vector<int32_t>> discard_readers;
  // Alg. 1: the clusters in execution order and their costs (ms, from
  // the performance tables); one cluster of every node for the other policies
  std::vector<std::vector<int>> clusters;
  std::vector<double> cluster_cost;
};

// comm.cpp: the strip halo exchange of `rank` on stream (cudaStream_t)
ktiler_status halo_exchange(ktiler_comm_s* c, int32_t rank, int32_t halo_rows, void* stream);

ktiler_status build_schedule(Graph& g, int64_t cache_bytes, const ktiler_fragment_policy& pol, Schedule& out);
ktiler_status build_schedule_core(Graph& g, int64_t cache_bytes, const ktiler_fragment_policy& pol, Schedule& out);
void compute_discards(const Graph& g, Schedule& s, std::vector<int32_t>* sub_of_block = nullptr);

}  // namespace kt
