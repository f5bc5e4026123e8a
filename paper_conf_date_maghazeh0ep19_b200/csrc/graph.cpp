// Graph store, validation and the affine footprint / dependency analyser
// (SURVEY §8(a) a1–a3).  The paper's block analyzer derives block dependencies and
// per-block memory lines from a SASSI memory trace; here each
// kernel declares its per-block footprint as affine maps and both products are
// computed in closed form:
//   - dependency: consumer block c depends on producer block p iff p's write rect
//     intersects c's read rect (byte-level RAW), which for rectangles
//     is an index interval per axis (Graph::producers / Graph::consumers);
//   - memory lines: the 128-B lines of each access's clipped rect.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <mutex>

#include "kt_internal.h"

struct ktiler_graph_s {
  kt::Graph g;
};

namespace kt {

static thread_local std::string t_err;
void set_error(const std::string& m) { t_err = m; }
void clear_error() { t_err.clear(); }
ktiler_status fail(ktiler_status s, const std::string& m) {
  t_err = m;
  return s;
}
const char* last_error() { return t_err.c_str(); }

static PRect clip(int64_t x0, int64_t y0, int64_t x1, int64_t y1, int64_t W, int64_t H) {
  PRect r{std::max<int64_t>(x0, 0), std::max<int64_t>(y0, 0), std::min(x1, W), std::min(y1, H)};
  return r;
}

PRect Graph::access_rect(int node, int acc, int64_t bx, int64_t by) const {
  const Access& a = nodes[node].acc[acc];
  const Buffer& b = bufs[a.buf];
  return clip(a.ax * bx + a.ox - a.hl, a.ay * by + a.oy - a.ht, a.ax * (bx + 1) + a.ox + a.hr,
              a.ay * (by + 1) + a.oy + a.hb, b.d.width, b.d.height);
}

// Indices i in [0, n) whose interval [a*i + o - hl, a*(i+1) + o + hr) meets [lo, hi).
static void hit_range(int64_t a, int64_t o, int64_t hl, int64_t hr, int64_t lo, int64_t hi, int64_t n, int64_t& i0,
                      int64_t& i1) {
  if (lo >= hi) {
    i0 = i1 = 0;
    return;
  }
  i0 = std::max<int64_t>(0, floordiv(lo - o - hr, a));
  i1 = std::min<int64_t>(n, floordiv(hi - o + hl - 1, a) + 1);
  if (i1 < i0) i1 = i0;
}

BRange Graph::producers(const Chan& c, int64_t bx, int64_t by) const {
  PRect rr = access_rect(c.v, c.r, bx, by);
  const Node& u = nodes[c.u];
  const Access& w = u.acc[c.w];
  BRange out{0, 0, 0, 0};
  if (rr.empty()) return out;
  hit_range(w.ax, w.ox, w.hl, w.hr, rr.x0, rr.x1, u.gx(), out.x0, out.x1);
  hit_range(w.ay, w.oy, w.ht, w.hb, rr.y0, rr.y1, u.gy(), out.y0, out.y1);
  return out;
}

BRange Graph::consumers(const Chan& c, int64_t px, int64_t py) const {
  PRect wr = access_rect(c.u, c.w, px, py);
  const Node& v = nodes[c.v];
  const Access& r = v.acc[c.r];
  BRange out{0, 0, 0, 0};
  if (wr.empty()) return out;
  hit_range(r.ax, r.ox, r.hl, r.hr, wr.x0, wr.x1, v.gx(), out.x0, out.x1);
  hit_range(r.ay, r.oy, r.ht, r.hb, wr.y0, wr.y1, v.gy(), out.y0, out.y1);
  return out;
}

// True stencil of each built-in, for the declared output tile (tw, th) of the WRITE
// access: read map (ax, ay, ox, oy, halos).  A declared read footprint must match it
// exactly, so a mis-declared footprint can never yield an invalid schedule.
static bool builtin_read_map(int op, const Access& w, Access& r, int radius = 0) {
  r.mode = KTILER_READ;
  r.ox = w.ox;
  r.oy = w.oy;
  r.ax = w.ax;
  r.ay = w.ay;
  r.hl = r.hr = r.ht = r.hb = 0;
  switch (op) {
    case KTILER_OP_GRAY:
    case KTILER_OP_THRESH: return true;
    case KTILER_OP_BLUR5: r.hl = r.hr = r.ht = r.hb = 2; return true;
    case KTILER_OP_SOBEL3: r.hl = r.hr = r.ht = r.hb = 1; return true;
    case KTILER_OP_DOWN2:
      r.ax = 2 * w.ax; r.ay = 2 * w.ay; r.ox = 2 * w.ox; r.oy = 2 * w.oy;
      return true;
    case KTILER_OP_JACOBI: r.hl = r.hr = 2; r.ht = r.hb = 1; return true;  // (u, v) of the 4 neighbours
    case KTILER_OP_GAUSS_F32: r.hl = r.hr = r.ht = r.hb = radius; return true;
    default: return false;
  }
}

static int builtin_in_elem(int op) {
  return op == KTILER_OP_GRAY ? 3 : ((op == KTILER_OP_THRESH || op == KTILER_OP_JACOBI || op == KTILER_OP_GAUSS_F32) ? 4 : 1);
}
static int builtin_out_elem(int op) {
  return (op == KTILER_OP_SOBEL3 || op == KTILER_OP_JACOBI || op == KTILER_OP_GAUSS_F32) ? 4 : 1;
}

ktiler_status Graph::finalize() {
  if (finalized) return KTILER_OK;
  const int nn = (int)nodes.size();
  if (nn == 0) return fail(KTILER_E_INVALID, "graph has no kernels");
  for (auto& b : bufs) {
    b.writer = -1;
    b.readers.clear();
  }
  for (int i = 0; i < nn; ++i) {
    for (auto& a : nodes[i].acc) {
      if (a.mode == KTILER_WRITE) {
        if (bufs[a.buf].writer >= 0 && bufs[a.buf].writer != i)
          return fail(KTILER_E_INVALID, "buffer " + std::to_string(a.buf) + " written by two kernels (no buffer reuse, SURVEY A20)");
        bufs[a.buf].writer = i;
      }
    }
  }
  for (int i = 0; i < nn; ++i)
    for (auto& a : nodes[i].acc)
      if (a.mode == KTILER_READ) {
        if (bufs[a.buf].writer == i) return fail(KTILER_E_INVALID, "kernel " + std::to_string(i) + " reads its own output (intra-kernel deps are not allowed, PAPER.md:189)");
        bufs[a.buf].readers.push_back(i);
      }
  // channels (implied by footprints); every declared edge must be one of them
  in_ch.assign(nn, {});
  out_ch.assign(nn, {});
  for (int v = 0; v < nn; ++v)
    for (int r = 0; r < (int)nodes[v].acc.size(); ++r) {
      const Access& a = nodes[v].acc[r];
      if (a.mode != KTILER_READ) continue;
      int u = bufs[a.buf].writer;
      if (u < 0) continue;  // external input
      int w = -1;
      for (int k = 0; k < (int)nodes[u].acc.size(); ++k)
        if (nodes[u].acc[k].mode == KTILER_WRITE && nodes[u].acc[k].buf == a.buf) w = k;
      Chan c{v, r, u, w, a.buf};
      if (nodes[u].gz() != nodes[v].gz())
        return fail(KTILER_E_INVALID, "kernels " + std::to_string(u) + " and " + std::to_string(v) + " disagree on frames (grid.z)");
      in_ch[v].push_back(c);
      out_ch[u].push_back(c);
    }
  for (auto& e : edges) {
    bool ok = false;
    for (auto& c : in_ch[e.dst]) ok |= (c.u == e.src && c.buf == e.buf);
    if (!ok) return fail(KTILER_E_INVALID, "edge " + std::to_string(e.src) + "->" + std::to_string(e.dst) + " on buffer " + std::to_string(e.buf) + ": src does not write it or dst does not read it");
  }
  // topological order (Kahn, smallest id first -> deterministic)
  std::vector<int> indeg(nn, 0);
  std::vector<std::vector<int>> succ(nn);
  for (int v = 0; v < nn; ++v)
    for (auto& c : in_ch[v]) {
      bool dup = false;
      for (int s : succ[c.u]) dup |= (s == v);
      if (!dup) {
        succ[c.u].push_back(v);
        indeg[v]++;
      }
    }
  topo.clear();
  std::vector<int> ready;
  for (int v = 0; v < nn; ++v)
    if (!indeg[v]) ready.push_back(v);
  while (!ready.empty()) {
    auto it = std::min_element(ready.begin(), ready.end());
    int v = *it;
    ready.erase(it);
    topo.push_back(v);
    for (int s : succ[v])
      if (--indeg[s] == 0) ready.push_back(s);
  }
  if ((int)topo.size() != nn) return fail(KTILER_E_CYCLE, "kernel graph has a cycle (PAPER.md:153 assumes a DAG)");
  total_blocks = 0;
  for (auto& n : nodes) {
    n.gid0 = total_blocks;
    total_blocks += n.nblocks;
  }
  finalized = true;
  return KTILER_OK;
}

}  // namespace kt

using namespace kt;

extern "C" {

const char* ktiler_status_str(ktiler_status s) {
  switch (s) {
    case KTILER_OK: return "KTILER_OK";
    case KTILER_E_INVALID: return "KTILER_E_INVALID";
    case KTILER_E_CYCLE: return "KTILER_E_CYCLE";
    case KTILER_E_UNTILEABLE: return "KTILER_E_UNTILEABLE";
    case KTILER_E_NOMEM: return "KTILER_E_NOMEM";
    case KTILER_E_CUDA: return "KTILER_E_CUDA";
    case KTILER_E_STATE: return "KTILER_E_STATE";
    case KTILER_E_UNSUPPORTED: return "KTILER_E_UNSUPPORTED";
  }
  return "KTILER_E_UNKNOWN";
}

const char* ktiler_last_error(void) { return kt::last_error(); }
int32_t ktiler_abi_version(void) { return KTILER_ABI_VERSION; }

ktiler_status ktiler_graph_create(ktiler_graph_t* out) {
  if (!out) return fail(KTILER_E_INVALID, "out is NULL");
  try {
    *out = new ktiler_graph_s();
  } catch (...) {
    return fail(KTILER_E_NOMEM, "graph allocation failed");
  }
  clear_error();
  return KTILER_OK;
}

void ktiler_graph_destroy(ktiler_graph_t g) { delete g; }

ktiler_status ktiler_add_buffer(ktiler_graph_t g, const ktiler_buffer_desc* d, int32_t* buf_id) {
  if (!g || !d || !buf_id) return fail(KTILER_E_INVALID, "NULL argument");
  if (g->g.finalized) return fail(KTILER_E_STATE, "graph already planned; create a new graph");
  ktiler_buffer_desc b = *d;
  if (b.width <= 0 || b.height <= 0 || b.frames <= 0)
    return fail(KTILER_E_INVALID, "buffer sizes must be positive");
  if (b.elem_bytes != 1 && b.elem_bytes != 3 && b.elem_bytes != 4)
    return fail(KTILER_E_INVALID, "elem_bytes must be 1, 3 or 4");
  if (((uint64_t)b.base) & 127) return fail(KTILER_E_INVALID, "buffer base must be 128-B aligned (SURVEY A10)");
  if (b.pitch_bytes < b.width * b.elem_bytes || (b.pitch_bytes & 15))
    return fail(KTILER_E_INVALID, "pitch_bytes must be >= width*elem_bytes and a multiple of 16");
  if (b.frame_stride_bytes == 0) b.frame_stride_bytes = b.height * b.pitch_bytes;
  if (b.frame_stride_bytes < b.height * b.pitch_bytes || (b.frame_stride_bytes & 15))
    return fail(KTILER_E_INVALID, "frame_stride_bytes must be >= height*pitch_bytes and a multiple of 16");
  if (b.ring_frames < 0 || b.ring_frames >= b.frames) b.ring_frames = b.ring_frames < 0 ? -1 : 0;
  if (b.ring_frames < 0) return fail(KTILER_E_INVALID, "ring_frames must be >= 0");
  if (b.ring_frames && !(b.flags & KTILER_BUF_INTERNAL))
    return fail(KTILER_E_INVALID, "a ring buffer (ring_frames > 0) must be INTERNAL: its frames are overwritten");
  Buffer nb;
  nb.d = b;
  nb.addr = (uint64_t)b.base;
  const int64_t slots = b.ring_frames ? b.ring_frames : b.frames;
  nb.span = (slots - 1) * b.frame_stride_bytes + (b.height - 1) * b.pitch_bytes + b.width * b.elem_bytes;
  nb.line0 = (int64_t)(nb.addr >> 7);
  nb.nlines = (int64_t)((nb.addr + nb.span - 1) >> 7) - nb.line0 + 1;
  for (size_t i = 0; i < g->g.bufs.size(); ++i) {
    const Buffer& o = g->g.bufs[i];
    if (nb.addr < o.addr + o.span && o.addr < nb.addr + nb.span)
      return fail(KTILER_E_INVALID, "buffer overlaps buffer " + std::to_string(i) + " (aliasing, SURVEY A20)");
  }
  *buf_id = (int32_t)g->g.bufs.size();
  g->g.bufs.push_back(nb);
  clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_add_kernel(ktiler_graph_t g, const ktiler_kernel_desc* d, int32_t* node_id) {
  if (!g || !d || !node_id) return fail(KTILER_E_INVALID, "NULL argument");
  if (g->g.finalized) return fail(KTILER_E_STATE, "graph already planned; create a new graph");
  if (d->op < KTILER_OP_GRAY || d->op > KTILER_OP_GAUSS_F32) return fail(KTILER_E_INVALID, "unknown op");
  if (d->n_access <= 0 || !d->access) return fail(KTILER_E_INVALID, "a kernel needs at least one access");
  Node n;
  n.op = d->op;
  for (int k = 0; k < 3; ++k) {
    if (d->grid[k] == 0 || d->block[k] == 0) return fail(KTILER_E_INVALID, "grid/block dims must be >= 1");
    n.grid[k] = d->grid[k];
    n.block[k] = d->block[k];
  }
  n.nblocks = (int64_t)n.grid[0] * n.grid[1] * n.grid[2];
  const int nb = (int)g->g.bufs.size();
  for (int i = 0; i < d->n_access; ++i) {
    const ktiler_access& a = d->access[i];
    if (a.buf_id < 0 || a.buf_id >= nb) return fail(KTILER_E_INVALID, "access buffer id out of range");
    if (a.mode != KTILER_READ && a.mode != KTILER_WRITE) return fail(KTILER_E_INVALID, "access mode must be READ or WRITE");
    if (a.ax <= 0 || a.ay <= 0) return fail(KTILER_E_INVALID, "access ax, ay must be >= 1");
    if (a.halo_l < 0 || a.halo_r < 0 || a.halo_t < 0 || a.halo_b < 0) return fail(KTILER_E_INVALID, "halos must be >= 0");
    if ((int64_t)g->g.bufs[a.buf_id].d.frames != (int64_t)n.grid[2])
      return fail(KTILER_E_INVALID, "grid.z must equal the frames of every accessed buffer");
    Access x;
    x.buf = a.buf_id; x.mode = a.mode; x.ax = a.ax; x.ay = a.ay; x.ox = a.ox; x.oy = a.oy;
    x.hl = a.halo_l; x.hr = a.halo_r; x.ht = a.halo_t; x.hb = a.halo_b;
    if (x.mode == KTILER_WRITE) {
      if (n.wacc >= 0 && d->op != KTILER_OP_CUSTOM) return fail(KTILER_E_INVALID, "built-in kernels have exactly one WRITE access");
      n.wacc = i;
    } else {
      if (d->op == KTILER_OP_JACOBI && n.racc >= 0) {
        if (n.racc2 >= 0) return fail(KTILER_E_INVALID, "KTILER_OP_JACOBI has exactly two READ accesses");
        n.racc2 = i;
      } else {
        if (n.racc >= 0 && d->op != KTILER_OP_CUSTOM) return fail(KTILER_E_INVALID, "built-in kernels have exactly one READ access");
        n.racc = i;
      }
    }
    n.acc.push_back(x);
  }
  if (n.wacc < 0) return fail(KTILER_E_INVALID, "a kernel needs a WRITE access");
  if (d->params_bytes) {
    if (!d->params) return fail(KTILER_E_INVALID, "params is NULL");
    n.params.assign((const uint8_t*)d->params, (const uint8_t*)d->params + d->params_bytes);
  }
  const Access& w = n.acc[n.wacc];
  const Buffer& ob = g->g.bufs[w.buf];
  if ((int64_t)n.grid[0] * w.ax + w.ox < ob.d.width || (int64_t)n.grid[1] * w.ay + w.oy < ob.d.height)
    return fail(KTILER_E_INVALID, "grid does not cover the written buffer");
  if (d->op == KTILER_OP_CUSTOM) {
    if (!d->launch) return fail(KTILER_E_INVALID, "KTILER_OP_CUSTOM needs a launch function");
    n.launch = d->launch;
    n.user = d->user;
  } else {
    if (n.racc < 0) return fail(KTILER_E_INVALID, "built-in kernels have exactly one READ access");
    if (w.hl || w.hr || w.ht || w.hb || w.ox || w.oy)
      return fail(KTILER_E_INVALID, "built-in WRITE access must have zero offsets and halos (output tile = ax x ay)");
    if (d->op == KTILER_OP_GAUSS_F32) {  // sigma -> radius and f32 taps (f64-normalised, reading A43)
      float sigma = 0.0f;
      if (n.params.size() != sizeof(float)) return fail(KTILER_E_INVALID, "GAUSS_F32 params must be one float (sigma)");
      std::memcpy(&sigma, n.params.data(), sizeof(float));
      if (!(sigma > 0.0f) || std::ceil(3.0 * (double)sigma) > 4.0)
        return fail(KTILER_E_INVALID, "GAUSS_F32 sigma must be > 0 with ceil(3 sigma) <= 4");
      n.radius = (int)std::ceil(3.0 * (double)sigma);
      double wk[9], sum = 0.0;
      for (int k = -n.radius; k <= n.radius; ++k) sum += (wk[k + n.radius] = std::exp(-(double)k * k / (2.0 * sigma * sigma)));
      for (int k = 0; k <= 2 * n.radius; ++k) n.taps[k] = (float)(wk[k] / sum);
      n.T = sigma;
    }
    Access want;
    builtin_read_map(d->op, w, want, n.radius);
    const Access& r = n.acc[n.racc];
    // the declared footprint must cover the true stencil (same scale and offset, halos at
    // least the stencil's): a larger one only adds dependencies (e.g. the line-quantized
    // maps fitted from ktiler_discover_footprint), a smaller one could produce a wrong plan
    if (r.ax != want.ax || r.ay != want.ay || r.ox != want.ox || r.oy != want.oy || r.hl < want.hl ||
        r.hr < want.hr || r.ht < want.ht || r.hb < want.hb)
      return fail(KTILER_E_INVALID, "declared READ footprint does not cover the op's true stencil for its output tile");
    const Buffer& ib = g->g.bufs[r.buf];
    if (ib.d.elem_bytes != builtin_in_elem(d->op) || ob.d.elem_bytes != builtin_out_elem(d->op))
      return fail(KTILER_E_INVALID, "buffer element sizes do not match the op");
    if (d->op == KTILER_OP_JACOBI) {
      if (n.racc2 < 0) return fail(KTILER_E_INVALID, "KTILER_OP_JACOBI has exactly two READ accesses");
      const Access& c = n.acc[n.racc2];
      const Buffer& cb = g->g.bufs[c.buf];
      if (c.ax != 2 * w.ax || c.ay != w.ay || c.ox != 2 * w.ox || c.oy != w.oy)
        return fail(KTILER_E_INVALID, "KTILER_OP_JACOBI coefficient footprint must be (2*ax, ay) of the output's");
      if (cb.d.elem_bytes != 4 || cb.d.width != 2 * ob.d.width || cb.d.height != ob.d.height)
        return fail(KTILER_E_INVALID, "KTILER_OP_JACOBI coefficients are f32 [H][4W] (Ix, Iy, It, - per pixel)");
      if ((ob.d.width & 3) || (w.ax & 3)) return fail(KTILER_E_INVALID, "KTILER_OP_JACOBI needs an even image width and tile width");
      if (c.buf == r.buf || c.buf == w.buf) return fail(KTILER_E_INVALID, "KTILER_OP_JACOBI buffers must be distinct");
    }
    if (d->op == KTILER_OP_DOWN2) {
      if ((ib.d.width & 1) || (ib.d.height & 1)) return fail(KTILER_E_INVALID, "DOWN2 needs even input sizes (SURVEY A3)");
      if (ob.d.width != ib.d.width / 2 || ob.d.height != ib.d.height / 2)
        return fail(KTILER_E_INVALID, "DOWN2 output must be half the input size");
    } else if (ob.d.width != ib.d.width || ob.d.height != ib.d.height) {
      return fail(KTILER_E_INVALID, "input and output sizes differ");
    }
    if (d->op == KTILER_OP_THRESH || d->op == KTILER_OP_JACOBI) {
      if (n.params.size() != sizeof(float))
        return fail(KTILER_E_INVALID, "THRESH / JACOBI params must be one float (T / alpha^2)");
      std::memcpy(&n.T, n.params.data(), sizeof(float));
    }
    int64_t nt = n.nthreads();
    if (nt > 1024) return fail(KTILER_E_INVALID, "more than 1024 threads per block");
    n.scalar = (nt == w.ax * w.ay) && d->op != KTILER_OP_JACOBI && d->op != KTILER_OP_GAUSS_F32;
    if (d->op == KTILER_OP_GAUSS_F32 && w.ax > 248) return fail(KTILER_E_INVALID, "GAUSS_F32 tile width must be <= 248");
    if (!n.scalar) {
      if (w.ax % 16) return fail(KTILER_E_INVALID, "vector variant needs tile width % 16 == 0 (else use one thread per pixel)");
      if (nt % 32) return fail(KTILER_E_INVALID, "vector variant needs a multiple of 32 threads per block");
    }
  }
  *node_id = (int32_t)g->g.nodes.size();
  g->g.nodes.push_back(std::move(n));
  clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_add_edge(ktiler_graph_t g, int32_t src, int32_t dst, int32_t buf, float weight) {
  if (!g) return fail(KTILER_E_INVALID, "NULL graph");
  if (g->g.finalized) return fail(KTILER_E_STATE, "graph already planned; create a new graph");
  int nn = (int)g->g.nodes.size();
  if (src < 0 || src >= nn || dst < 0 || dst >= nn || buf < 0 || buf >= (int)g->g.bufs.size())
    return fail(KTILER_E_INVALID, "edge ids out of range");
  bool w = false, r = false;
  for (auto& a : g->g.nodes[src].acc) w |= (a.mode == KTILER_WRITE && a.buf == buf);
  for (auto& a : g->g.nodes[dst].acc) r |= (a.mode == KTILER_READ && a.buf == buf);
  if (!w || !r) return fail(KTILER_E_INVALID, "edge buffer must be written by src and read by dst");
  g->g.edges.push_back({src, dst, buf, weight});
  clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_set_perf_table(ktiler_graph_t g, int32_t node, int32_t npts, const int64_t* nb, const double* cold,
                                    const double* hot) {
  if (!g || !nb || !cold || !hot) return fail(KTILER_E_INVALID, "NULL argument");
  if (node < 0 || node >= (int)g->g.nodes.size()) return fail(KTILER_E_INVALID, "node out of range");
  if (npts < 1) return fail(KTILER_E_INVALID, "a performance table needs at least one point");
  for (int k = 0; k < npts; ++k) {
    if (nb[k] < 1 || (k && nb[k] <= nb[k - 1])) return fail(KTILER_E_INVALID, "block counts must be positive and increasing");
    if (!(cold[k] >= 0) || !(hot[k] >= 0)) return fail(KTILER_E_INVALID, "times must be >= 0");
  }
  Node& n = g->g.nodes[node];
  n.perf_n.assign(nb, nb + npts);
  n.perf_cold.assign(cold, cold + npts);
  n.perf_hot.assign(hot, hot + npts);
  clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_graph_block_deps(ktiler_graph_t g, int32_t node, int32_t bx, int32_t by, int32_t bz, int32_t* out,
                                      int64_t cap, int64_t* n) {
  if (!g || !n) return fail(KTILER_E_INVALID, "NULL argument");
  ktiler_status s = g->g.finalize();
  if (s) return s;
  const Graph& G = g->g;
  if (node < 0 || node >= (int)G.nodes.size()) return fail(KTILER_E_INVALID, "node out of range");
  const Node& v = G.nodes[node];
  if (bx < 0 || by < 0 || bz < 0 || bx >= v.gx() || by >= v.gy() || bz >= v.gz()) return fail(KTILER_E_INVALID, "block out of range");
  int64_t k = 0;
  for (auto& c : G.in_ch[node]) {
    BRange r = G.producers(c, bx, by);
    for (int64_t y = r.y0; y < r.y1; ++y)
      for (int64_t x = r.x0; x < r.x1; ++x) {
        if (out && k < cap) {
          out[4 * k] = c.u; out[4 * k + 1] = (int32_t)x; out[4 * k + 2] = (int32_t)y; out[4 * k + 3] = bz;
        }
        ++k;
      }
  }
  *n = k;
  clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_graph_block_lines(ktiler_graph_t g, int32_t node, int32_t bx, int32_t by, int32_t bz, int64_t* out,
                                       int64_t cap, int64_t* n) {
  if (!g || !n) return fail(KTILER_E_INVALID, "NULL argument");
  ktiler_status s = g->g.finalize();
  if (s) return s;
  const Graph& G = g->g;
  if (node < 0 || node >= (int)G.nodes.size()) return fail(KTILER_E_INVALID, "node out of range");
  const Node& v = G.nodes[node];
  if (bx < 0 || by < 0 || bz < 0 || bx >= v.gx() || by >= v.gy() || bz >= v.gz()) return fail(KTILER_E_INVALID, "block out of range");
  std::vector<int64_t> ls;
  for (int a = 0; a < (int)v.acc.size(); ++a)
    G.for_each_line_range(node, a, bx, by, bz, [&](int, int64_t l0, int64_t l1) {
      for (int64_t l = l0; l < l1; ++l) ls.push_back(l);
    });
  std::sort(ls.begin(), ls.end());
  ls.erase(std::unique(ls.begin(), ls.end()), ls.end());
  for (int64_t i = 0; i < (int64_t)ls.size() && i < cap; ++i)
    if (out) out[i] = ls[i];
  *n = (int64_t)ls.size();
  clear_error();
  return KTILER_OK;
}

}  // extern "C"

namespace kt {
Graph* graph_of(ktiler_graph_t g) { return g ? &g->g : nullptr; }
}
