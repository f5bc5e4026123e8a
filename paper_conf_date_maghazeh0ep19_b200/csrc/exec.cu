// Sub-kernel launcher and the plan/execute half of the C ABI.
//
// The paper enforces its schedule "by slightly modifying the source code" so that each
// sub-kernel launches only its subset of blocks.  Here a sub-kernel is a
// launch of the op's kernel over a 1-D grid whose blocks map to a list of <= 4 block
// rects (kernel parameter), so a ragged Alg. 2 fragment is still one launch.  The
// inter-launch gap the paper measures is removed by:
//   GRAPH       the launch sequence captured once into a CUDA graph (one host call);
//   PF_PDL      programmatic dependent launch: the next sub-kernel's CTAs are scheduled
//               while the previous one drains and wait in griddepcontrol.wait;
//   PERSISTENT  one launch; CTAs take tiles in schedule order from an atomic ticket and
//               wait on per-block completion flags (acquire/release at gpu scope) —
//               deadlock-free because producers always precede consumers in the order.
// Dead intermediate lines (last reader done) are dropped from L2 with discard.global.L2
// (no write-back): as the prologue of the next launch (stream/graph modes) or by the
// last reader tile (persistent mode).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <cstring>

#include "flow.cuh"
#include "kernels.cuh"
#include "kt_internal.h"

namespace kt {
Graph* graph_of(ktiler_graph_t g);
}

namespace {

using ktd::DBuf;
constexpr int MAXR = 4, MAXD = 8;
constexpr int KMAXST = 4;  // staging ring depth of the op kernels (KParams::nstage)
constexpr int PCOMP_WARPS = 4;  // compute warps per persistent CTA (+ producer + publisher warp)
constexpr int PCOMP_THREADS = 32 * PCOMP_WARPS;
constexpr int PSTAGES_MAX = 12;   // staging ring depth (slots that fit the CTA's share of smem)
constexpr int PERSIST_GROUPS_DEFAULT = 2;
constexpr int PMAX_NODES = 8;

struct LRect {
  int32_t x0, y0, z0, x1, y1, z1;
};
struct DRect {  // whole 128-B lines: row r -> base + (z mod ring)*fs + y*pitch + lb0 + k*128, k < lpr
  uint8_t* base;
  int64_t pitch, fstride, lb0, lpr;
  int32_t y0, y1, z0, z1;
  int32_t ring, pad;
};
__device__ __forceinline__ int64_t drect_zoff(const DRect& d, int64_t z) {
  return (d.ring ? (int64_t)((uint32_t)z % (uint32_t)d.ring) : z) * d.fstride;
}
// Device-side trace buffer (ktiler_trace_enable): NULL rec = tracing off.  Sharded by CTA
// and SM (TRACE_SHARDS counters, each owning cap records), so a record costs an atomic on
// one of many counters instead of one device-wide counter that every CTA of the step contends on
// (that serialisation slowed a traced 64 x 8K step by ~1.7 ms and penalised plans with
// many small CTAs).  ktiler_trace_read gathers the shards.
constexpr int TRACE_SHARDS = 256;
static_assert(TRACE_SHARDS == ktflow::FL_TRACE_SHARDS, "FLOW writes the same sharded trace layout");
struct TraceBuf {
  ktiler_trace_record* rec;
  unsigned long long* n;  // TRACE_SHARDS counters
  int64_t cap;            // records per shard
};
__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void trace_put(const TraceBuf& tb, uint64_t id, uint32_t kind, uint64_t t0, uint64_t t1) {
  uint32_t sm;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
  // shard by a hash of (record id, CTA, SM): small launches fill the low SM ids with
  // low CTA indices first, so SM or CTA alone would crowd a few shards
  const uint32_t sh =
      ((blockIdx.x * 0x9E3779B9u) ^ (sm * 0x85EBCA6Bu) ^ ((uint32_t)id * 0xC2B2AE35u)) >> 24 & (TRACE_SHARDS - 1);
  const unsigned long long k = atomicAdd(tb.n + sh, 1ull);
  if ((int64_t)k < tb.cap) tb.rec[(int64_t)sh * tb.cap + (int64_t)k] = ktiler_trace_record{id, sm, kind, t0, t1};
}

struct KParams {
  CUtensorMap tmap;     // input tile map (tensor TMA), valid if use_tmap
  TraceBuf tb;
  int64_t lid;          // launch index (trace id)
  uint32_t box_bytes;   // bytes one tensor-TMA box delivers
  int32_t use_tmap;
  int32_t in_stream;    // load the input evict-first (graph input; consumed intermediate of a tiled plan)
  DBuf in, out;
  DBuf aux;             // KTILER_OP_JACOBI: the coefficient buffer (second READ access)
  int32_t tw, th;
  float T;
  float taps[2 * ktd::GAUSS_H + 1];  // KTILER_OP_GAUSS_F32: f32 weights, taps[k + radius]
  int32_t radius;
  int32_t cdisc;  // KTILER_PF_CONSUMER_DISCARD: drop this block's (exclusively read) input lines once staged
  // KTILER_PF_HALO_DISCARD (blur5, sobel3 reads with halo): per producer block a reader
  // count; the reader that completes it drops the producer block's lines (uses the chain map
  // fields rax..way / pgx, pgy for the producer range)
  unsigned int* hcnt;       // [frames][pgy][pgx] readers so far (reset to 0 by the last one)
  const uint8_t* hneed;     // [pgy][pgx] consumer blocks reading each producer block
  int32_t nrect, ndisc, pdl;
  int64_t stage_bytes;  // one staging buffer (slot) of the ring
  int32_t nstage;       // ring depth (2..KMAXST)
  int32_t pad_ns;
  LRect r[MAXR];
  int64_t rpre[MAXR + 1];
  DRect d[MAXD];
  int64_t dpre[MAXD + 1];
  // GRAPH_CHAIN: per-block epoch flags and launch completion (see chain_* below)
  int32_t chain;           // 1: flag-synchronised PDL chain
  int32_t gx, gy;          // this node's grid (block linear index -> flag)
  int32_t pgx, pgy;        // producer node's grid (0: graph input, nothing to wait on)
  int32_t rax, ray, rox, roy, rhl, rhr, rht, rhb;  // read footprint (affine map)
  int32_t wax, way;        // producer write footprint
  unsigned int* flags;     // this node's block flags
  const unsigned int* pflags;  // producer node's block flags
  const unsigned int* epoch;   // current execute's epoch
  unsigned int* dcount;    // this launch's finished-CTA counter
  unsigned int* prefix;    // prefix[l] == epoch <=> launches 0..l all finished (this one at [0])
  const unsigned int* disc_prefix;  // discards may run once *disc_prefix == epoch
};

__device__ __forceinline__ unsigned int ld_acquire(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(unsigned int* p, unsigned int v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// Watchdog for every spin on another CTA's progress (CHAIN flags and prefixes, PERSISTENT
// counters): sleep between polls, and after KT_SPIN_LIMIT polls (seconds) trap with the
// waiter's identity in the message instead of hanging the GPU — an unsatisfiable wait is
// a schedule bug (every executor's order is deadlock-free by construction).
constexpr unsigned long long KT_SPIN_LIMIT = 1ull << 25;
__device__ __noinline__ void kt_watchdog_trap(const char* what, long long id, unsigned long long n) {
  printf("libktiler watchdog: %s (id %lld) waited %llu polls: trapping\n", what, id, n);
  __trap();
}
__device__ __forceinline__ void kt_spin(unsigned long long& n, unsigned ns, const char* what, long long id) {
  __nanosleep(ns);
  if (++n > KT_SPIN_LIMIT) kt_watchdog_trap(what, id, n);
}

// GRAPH_CHAIN, one warp: wait until every producer block of output block (bx, by, bz)
// has published this epoch.  Producer range = closed form of the affine footprints
// (SURVEY §8(a) a3), the same one the planner uses.
__device__ __forceinline__ void chain_wait(const KParams& p, int bx, int by, int bz, unsigned epoch, int lane) {
  if (p.pgx == 0) return;
  const int rx0 = max(0, p.rax * bx + p.rox - p.rhl), rx1 = min((int)p.in.W, p.rax * (bx + 1) + p.rox + p.rhr);
  const int ry0 = max(0, p.ray * by + p.roy - p.rht), ry1 = min((int)p.in.H, p.ray * (by + 1) + p.roy + p.rhb);
  const int px0 = rx0 / p.wax, px1 = min(p.pgx, (rx1 + p.wax - 1) / p.wax);
  const int py0 = ry0 / p.way, py1 = min(p.pgy, (ry1 + p.way - 1) / p.way);
  const int pw = px1 - px0, n = pw * (py1 - py0);
  for (int i = lane; i < n; i += 32) {
    const int dy = i / pw;
    const unsigned int* f = p.pflags + ((int64_t)bz * p.pgy + py0 + dy) * p.pgx + px0 + (i - dy * pw);
    for (unsigned long long w = 0; ld_acquire(f) != epoch;) kt_spin(w, 64, "CHAIN producer-block flag", (long long)(f - p.pflags));
  }
  __syncwarp();
}

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_launch() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ void do_discards(const KParams& p) {
  const int64_t total = p.dpre[p.ndisc];
  const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += nthr) {
    int k = 0;
    while (k + 1 < p.ndisc && i >= p.dpre[k + 1]) ++k;
    const DRect& d = p.d[k];
    int64_t j = i - p.dpre[k];
    int64_t row = j / d.lpr, l = j % d.lpr;
    int64_t h = d.y1 - d.y0;
    int64_t z = d.z0 + row / h, y = d.y0 + row % h;
    ktd::discard_line(d.base + drect_zoff(d, z) + y * d.pitch + d.lb0 + 128 * l);
  }
}

// Tile i of a launch: its rect list maps the launch's linear tile index to a block.
__device__ __forceinline__ ktd::Tile launch_tile(const KParams& p, int64_t lin64) {
  int k = 0;
  while (k + 1 < p.nrect && lin64 >= p.rpre[k + 1]) ++k;
  const LRect& r = p.r[k];
  // 32-bit index math (a launch has < 2^31 blocks): 64-bit division is ~100 instructions
  const unsigned lin = (unsigned)(lin64 - p.rpre[k]);
  const unsigned w = (unsigned)(r.x1 - r.x0), h = (unsigned)(r.y1 - r.y0);
  const unsigned q = lin / w, q2 = q / h;
  const int64_t bx = r.x0 + (int)(lin - q * w), by = r.y0 + (int)(q - q2 * h), bz = r.z0 + (int)q2;
  ktd::Tile t;
  t.z = bz;
  t.x0 = p.tw * bx;
  t.y0 = p.th * by;
  t.x1 = min(t.x0 + p.tw, p.out.W);
  t.y1 = min(t.y0 + p.th, p.out.H);
  t.fw = p.tw;
  t.pad = (int)(((unsigned)bz * (unsigned)p.gy + (unsigned)by) * (unsigned)p.gx + (unsigned)bx);  // block index
  return t;
}

// GRAPH_CHAIN: publish output block t.pad of this node, after a CTA barrier.  bar.sync
// orders every thread's tile writes before this thread's gpu-scope release (PTX memory
// model: release is cumulative over writes that precede it in causality order), so the
// consumer's acquire of the flag sees the whole tile — no separate fence.
__device__ __forceinline__ void chain_publish(const KParams& p, const ktd::Tile& t, unsigned epoch) {
  st_release(p.flags + t.pad, epoch);
}

// GRAPH_CHAIN end of CTA (thread 0): count it; the last CTA of the launch waits for the
// previous launches (prefix[-1]) and publishes prefix[0] — "launches 0..this all done".
__device__ __forceinline__ void chain_finish(const KParams& p, unsigned epoch, bool first_launch) {
  // relaxed: the count only says "this CTA's reads are consumed" (they were, before the
  // barrier); data visibility travels through the block flags
  const unsigned old = atomicAdd(p.dcount, 1u);
  if (old == gridDim.x - 1) {
    *p.dcount = 0;  // ready for the next execute (every CTA of this launch has counted)
    if (!first_launch)
      for (unsigned long long w = 0; ld_acquire(p.prefix - 1) != epoch;) kt_spin(w, 128, "CHAIN launch prefix", 0);
    __threadfence();
    st_release(p.prefix, epoch);
  }
}

// KTILER_PF_CONSUMER_DISCARD: the whole 128-B lines of this block's input rect (no halo,
// the buffer's only reader) leave L2 unwritten once they are staged in shared memory.
template <int OP>
__device__ __forceinline__ void consumer_discard(const KParams& p, const ktd::Tile& t, int nt, int tid) {
  constexpr int EB = OP == 2 ? 2 : 4;  // input bytes per output pixel along x (down2: 2 u8; thresh: 1 f32)
  const int64_t y0 = OP == 2 ? 2 * t.y0 : t.y0, nrows = OP == 2 ? 2 * (t.y1 - t.y0) : t.y1 - t.y0;
  const uint8_t* base = p.in.p + ktd::zoff(p.in, t.z);
  const int64_t b0 = EB * t.x0, b1 = EB * t.x1;
  // lines of row r: [ceil(a / 128), floor(b / 128)) of absolute addresses a, b; the count is
  // the same for every row (128-B pitch).  CTA-uniform set-up once, then 32-bit index math
  // per line (a 64-bit division per line cost more instructions than the down2 tile itself)
  const int64_t r0 = (int64_t)(uintptr_t)(base + y0 * p.in.pitch);
  const int64_t first = (r0 + b0 + 127) >> 7, last = (r0 + b1) >> 7;
  if (last <= first) return;
  const unsigned per = (unsigned)(last - first), n = per * (unsigned)nrows;
  const int64_t pitch = p.in.pitch;
  auto line = [&](unsigned r, unsigned l) {
    const int64_t row = r0 + (int64_t)r * pitch;
    ktd::discard_line(reinterpret_cast<const void*>((((row + b0 + 127) >> 7) + (int64_t)l) << 7));
  };
  if ((per & (per - 1)) == 0) {
    const int sh = __ffs(per) - 1;
    for (unsigned i = tid; i < n; i += nt) line(i >> sh, i & (per - 1));
  } else {
    for (unsigned i = tid; i < n; i += nt) {
      const unsigned r = i / per;
      line(r, i - r * per);
    }
  }
}

// Halo reads (blur5 of gray, sobel3 of down): a producer block's lines are dead once every
// consumer block whose declared footprint covers it has staged them.  Warp 0 counts this
// block in for each producer block in its range (closed form of the affine maps, as
// chain_wait); the reader that completes a count resets it and drops that block's lines.
__device__ __forceinline__ void halo_discard(const KParams& p, const ktd::Tile& t, int lane) {
  const int bx = (int)(t.x0 / p.tw), by = (int)(t.y0 / p.th), bz = (int)t.z;
  const int rx0 = max(0, p.rax * bx + p.rox - p.rhl), rx1 = min((int)p.in.W, p.rax * (bx + 1) + p.rox + p.rhr);
  const int ry0 = max(0, p.ray * by + p.roy - p.rht), ry1 = min((int)p.in.H, p.ray * (by + 1) + p.roy + p.rhb);
  const int px0 = rx0 / p.wax, px1 = min(p.pgx, (rx1 + p.wax - 1) / p.wax);
  const int py0 = ry0 / p.way, py1 = min(p.pgy, (ry1 + p.way - 1) / p.way);
  const int pw = px1 - px0, n = pw * (py1 - py0);
  const uint8_t* fb = p.in.p + ktd::zoff(p.in, bz);
  const unsigned upw = (unsigned)max(pw, 1);
  for (int i0 = 0; i0 < n; i0 += 32) {
    const int i = i0 + lane;
    const unsigned qd = (unsigned)i / upw;
    const int py = py0 + (int)qd, px = px0 + (int)((unsigned)i - qd * upw);
    bool last = false;
    if (i < n) {
      const int64_t idx = ((int64_t)bz * p.pgy + py) * p.pgx + px;
      last = atomicAdd(p.hcnt + idx, 1u) + 1u == (unsigned)p.hneed[(int64_t)py * p.pgx + px];
      if (last) p.hcnt[idx] = 0u;  // every reader of this execute has counted: ready for the next one
    }
    // the whole warp drops each completed producer block's lines (u8 input: bytes = pixels)
    for (unsigned m = __ballot_sync(0xFFFFFFFFu, last); m; m &= m - 1) {
      const int src = __ffs(m) - 1;
      const int qy = __shfl_sync(0xFFFFFFFFu, py, src), qx = __shfl_sync(0xFFFFFFFFu, px, src);
      const int64_t x0 = (int64_t)p.wax * qx, x1 = min((int64_t)p.in.W, x0 + p.wax);
      const int64_t y0 = (int64_t)p.way * qy, y1 = min((int64_t)p.in.H, y0 + p.way);
      const int64_t a0 = (int64_t)(uintptr_t)(fb + y0 * p.in.pitch + x0);
      const int64_t l0 = (a0 + 127) >> 7, l1 = (a0 + (x1 - x0)) >> 7;  // whole lines of the first row
      if (l1 <= l0) continue;
      // 32-bit index math per line (as consumer_discard): shift / mask for power-of-two rows
      const unsigned per = (unsigned)(l1 - l0), tot = per * (unsigned)(y1 - y0);
      const bool pow2 = (per & (per - 1)) == 0;
      const int sh = __ffs(per) - 1;
      for (unsigned k = lane; k < tot; k += 32) {
        const unsigned r = pow2 ? k >> sh : k / per, l = k - r * per;
        ktd::discard_line(reinterpret_cast<const void*>(((l0 + (int64_t)l) << 7) + (int64_t)r * p.in.pitch));
      }
    }
  }
}

// NST: staging ring depth; 2 (compile time, the default code path) or 0 = p.nstage at run
// time (KTILER_STAGES variants of the L2-fed consumers, instantiated for down2 / sobel3 /
// thresh only)
// LEAN: no GRAPH_CHAIN flags, no counted halo discards, no tracing, no discard lists, tensor-
// map staging (the launch has none of the former; launch_fn picks it): those paths are compiled out, which leaves the register
// allocator more room (blur5 runs at its 80-register cap)
template <int OP, bool SCALAR, int NST = 2, bool LEAN = false>
__global__ void __launch_bounds__(256, (OP == 3 || OP == 6 || OP == 7) ? 2 : (OP == 1 ? 3 : 4)) op_kernel(const __grid_constant__ KParams p) {
  __shared__ uint64_t s_t0;  // trace: CTA start (kept out of registers)
  __shared__ uint64_t s_tr, s_tl;  // trace: producers ready (after PDL wait), first tile staged
  __shared__ unsigned int s_epoch;
  const int nt = blockDim.x * blockDim.y * blockDim.z;
  const int tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  if (tid == 0) {
    if ((!LEAN && p.tb.rec)) s_t0 = gtimer();
    if ((!LEAN && p.chain)) s_epoch = *(volatile const unsigned int*)p.epoch;
  }
  // PDL (p.pdl): wait for the programmatic producers (griddepcontrol.wait), then let this
  // launch's dependents be scheduled (p.pdl == 1: right away; 2: only when CTAs exit).  The
  // vector path sets up its shared-memory ring first, so that part overlaps the wait.
  // p.pdl == 3: a source sub-kernel whose only programmatic edge is a dispatch-order edge
  // (dag_order_node): it reads no producer's output, so it does not wait for one
  auto pdl_enter = [&]() {
    if (p.pdl && (p.pdl != 3 || p.ndisc)) pdl_wait();
    if (!LEAN && p.ndisc) do_discards(p);  // LEAN launches carry no discard lists
    if (p.pdl == 1 || p.pdl == 3) pdl_launch();
  };
  if ((!LEAN && p.chain)) {
    pdl_launch();  // the next sub-kernel may become resident now: it waits on tile flags
  } else if (SCALAR) {
    pdl_enter();
  }
  const int64_t ntiles = p.rpre[p.nrect];
  if (SCALAR) {
    __syncthreads();
    const unsigned epoch = s_epoch;
    for (int64_t i = blockIdx.x; i < ntiles; i += gridDim.x) {
      const ktd::Tile t = launch_tile(p, i);
      if ((!LEAN && p.chain)) {
        if (tid < 32) chain_wait(p, (int)(t.x0 / p.tw), (int)(t.y0 / p.th), (int)t.z, epoch, tid);
        __syncthreads();
      }
      ktd::scalar_tile(OP, p.in, p.out, t, p.T, nt, tid);
      if ((!LEAN && p.chain)) {
        __syncthreads();
        if (tid == 0) chain_publish(p, t, epoch);
      }
    }
  } else {
    // Grid-stride over the launch's tiles with a ring of S = p.nstage shared buffers (2 by
    // default; deeper for L2-fed sub-kernels, KTILER_STAGES): the TMA copies of the next
    // S - 1 tiles stream in while one computes.
    extern __shared__ __align__(128) uint8_t ktsm[];
    __shared__ __align__(8) uint64_t mbar[KMAXST];
    __shared__ ktd::Tile s_tile[KMAXST];  // decoded once by warp 0, read by all after the mbarrier
    __shared__ uint64_t s_tw[KMAXST];     // trace (chain): producers ready
    const int S = NST ? NST : (p.nstage < 2 ? 2 : (p.nstage > KMAXST ? KMAXST : p.nstage));
    const int64_t i0 = blockIdx.x;
    unsigned epoch = 0;
    auto issue = [&](int64_t i, int slot) {  // warp 0
      const ktd::Tile t = launch_tile(p, i);
      if ((!LEAN && p.chain)) {  // producers' tiles complete (acquire), then hand them to the async proxy
        chain_wait(p, (int)(t.x0 / p.tw), (int)(t.y0 / p.th), (int)t.z, epoch, tid);
        ktd::fence_proxy_async();
        if ((!LEAN && p.tb.rec) && tid == 0) s_tw[slot] = gtimer();
      }
      uint8_t* dst = ktsm + slot * p.stage_bytes;
      if (LEAN || p.use_tmap) {  // LEAN launches always stage by tensor map
        if (tid == 0) {
          s_tile[slot] = t;
          ktd::stage_issue_tmap(OP, &p.tmap, p.box_bytes, p.in, t, dst, &mbar[slot], p.in_stream != 0);
        }
      } else if constexpr (!LEAN) {
        if (tid == 0) s_tile[slot] = t;
        ktd::stage_issue(OP, p.in, t, dst, &mbar[slot], tid);
      }
    };
    // Tensor-map staging (one thread issues): thread 0 waits for the programmatic producers
    // itself (griddepcontrol.wait orders the executing thread after every prerequisite
    // grid's completion and memory flush) and requests the CTA's first tile at once,
    // instead of after every warp of the CTA has reached the barrier (64 x 8K: -0.7% tiled
    // and untiled).  The other threads still pass pdl_enter before touching
    // anything a producer wrote; they read only the staged tile, after its mbarrier.
    const bool early = (LEAN || p.use_tmap) && !(!LEAN && p.chain) && i0 < ntiles;
    if (tid == 0) {
      for (int j = 0; j < S; ++j) ktd::mbar_init(&mbar[j], 1);
      ktd::fence_proxy_async();
      if (early) {
        if (p.pdl && (p.pdl != 3 || p.ndisc)) pdl_wait();
        issue(i0, 0);
      }
    }
    __syncthreads();
    if (!(!LEAN && p.chain)) pdl_enter();
    if ((!LEAN && p.tb.rec) && tid == 0) s_tr = gtimer();
    epoch = s_epoch;
    if (tid < 32)
      for (int j = early ? 1 : 0; j < S && i0 + j * (int64_t)gridDim.x < ntiles; ++j) issue(i0 + j * (int64_t)gridDim.x, j);
    int b = 0;          // slot of the current tile
    unsigned par = 0;   // its mbarrier phase parity (flips each time the ring wraps)
    for (int64_t i = i0; i < ntiles; i += gridDim.x) {
      uint8_t* buf = ktsm + b * p.stage_bytes;
      ktd::mbar_wait(&mbar[b], par);
      if ((!LEAN && p.tb.rec) && tid == 0 && i == i0) s_tl = gtimer();
      const ktd::Tile t = s_tile[b];
      if constexpr (OP == 2 || OP == 4) {
        if (p.cdisc) consumer_discard<OP>(p, t, nt, tid);
      }
      if constexpr (OP == 1 || OP == 3) {  // as soon as staged: the earlier, the fewer write-backs
        if ((!LEAN && p.hcnt) && tid < 32) halo_discard(p, t, tid);
      }

      if ((OP == 1 || OP == 3 || OP == 6 || OP == 7) && ktd::needs_fix(OP, p.in, t)) {
        ktd::stage_fix(OP, p.in, t, buf, nt, tid);
        __syncthreads();
      }
      ktd::compute_tile(OP, p.out, t, buf, p.T, nt, tid, &p.aux, p.taps, p.radius);
      const int64_t nx = i + (int64_t)S * gridDim.x;
      if ((!LEAN && p.chain)) {
        __syncthreads();  // tile written (and buffer b consumed)
        if (tid == 0) {
          const uint64_t tc = (!LEAN && p.tb.rec) ? gtimer() : 0;
          chain_publish(p, t, epoch);
          if ((!LEAN && p.tb.rec)) {
            trace_put(p.tb, p.lid, 3, s_tw[b], tc);  // producers ready -> tile computed
            trace_put(p.tb, p.lid, 4, tc, gtimer());  // publish (fence + release)
          }
        }
      } else if (nx < ntiles) {
        __syncthreads();  // buffer b consumed
      }
      if (nx < ntiles && tid < 32) {
        ktd::fence_proxy_async();
        issue(nx, b);
      }
      if (++b == S) {
        b = 0;
        par ^= 1u;
      }
    }
  }
  if ((!LEAN && p.chain)) {
    __syncthreads();
    if (tid == 0) chain_finish(p, s_epoch, p.chain == 2);
    if (p.ndisc) {  // lines dead after an earlier launch: wait until it and all before it finished
      if (tid == 0)
        for (unsigned long long w = 0; ld_acquire(p.disc_prefix) != s_epoch;) kt_spin(w, 128, "CHAIN discard prefix", 0);
      __syncthreads();
      do_discards(p);
    }
  }
  if ((!LEAN && p.tb.rec)) {
    __syncthreads();
    if (tid == 0) {
      trace_put(p.tb, p.lid, 0, s_t0, gtimer());
      if (!SCALAR && !(!LEAN && p.chain) && blockIdx.x < ntiles) {  // CTA phases: start -> ready -> first tile staged
        trace_put(p.tb, p.lid, 5, s_t0, s_tr);
        trace_put(p.tb, p.lid, 6, s_tr, s_tl);
      }
    }
  }
}

// GRAPH_CHAIN tail (launched without PDL): wait until every launch of the chain finished
// (prefix of the last one), then retire the remaining dead lines.  The epoch is advanced by
// chain_epoch_kernel, stream-ordered after this one (a CTA of this kernel may start late
// and must still read the current epoch).
__global__ void chain_tail_kernel(const __grid_constant__ KParams p) {
  __shared__ unsigned int s_ep;
  if (threadIdx.x == 0) {
    s_ep = *(volatile const unsigned int*)p.epoch;
    for (unsigned long long w = 0; ld_acquire(p.disc_prefix) != s_ep;) kt_spin(w, 256, "CHAIN tail prefix", 0);
  }
  __syncthreads();
  if (p.ndisc) do_discards(p);
}

// ktiler_selftest(KTILER_SELFTEST_SQRT): the production sqrt2_int vs __fsqrt_rn.
__global__ void selftest_sqrt_kernel(unsigned n, unsigned long long* bad) {
  unsigned long long local = 0;
  for (unsigned i = 2 * (blockIdx.x * blockDim.x + threadIdx.x); i <= n; i += 2 * gridDim.x * blockDim.x) {
    const float a = (float)i, b = (float)(i + 1);
    const float2 r = ktd::sqrt2_int(make_float2(a, b));
    local += (__float_as_uint(r.x) != __float_as_uint(__fsqrt_rn(a))) +
             (i + 1 <= n && __float_as_uint(r.y) != __float_as_uint(__fsqrt_rn(b)));
  }
  if (local) atomicAdd(bad, local);
}

// GRAPH_CHAIN: advance the epoch (one thread), stream-ordered after the tail kernel.
__global__ void chain_epoch_kernel(unsigned int* epoch) { *epoch += 1u; }

__global__ void discard_kernel(const __grid_constant__ KParams p) {
  const uint64_t tt0 = p.tb.rec ? gtimer() : 0;
  if (p.pdl) pdl_wait();
  do_discards(p);
  if (p.pdl) pdl_launch();
  if (p.tb.rec) {
    __syncthreads();
    if (threadIdx.x == 0) trace_put(p.tb, p.lid, 0, tt0, gtimer());
  }
}

// ------------------------------------------------------------------------------------
// persistent executor
// ------------------------------------------------------------------------------------
// One launch runs the whole schedule.  The schedule's sub-kernels are replayed as a
// stream of tickets in a (skewed) total order that respects every dependency
// (PAPER.md:271): a ticket is one block (tile) of a sub-kernel, or one chunk of a discard
// list.  Ticket i belongs to CTA i mod G (static, no ticket atomics); the host lays each
// CTA's tickets out contiguously so a warp fetches 32 of them with one coalesced load.
// Synchronisation is per SUB-KERNEL, not per block: each sub-kernel (and each discard
// list) is a "group" whose tickets may start once the completion counters of the groups
// it depends on (Schedule::sub_deps, the block-level dependencies PAPER.md:173–193
// aggregated per sub-kernel; for discards: every reader of the lines) have reached
// epoch x their tile counts.  With the skewed order a consumer sub-kernel is issued about
// one pipeline step after its producer, so the check almost never waits; and a CTA
// re-checks only when its next ticket belongs to another group.
// Deadlock-free: a group's dependencies have all their tickets earlier in the order, so
// the smallest unfinished ticket is always runnable and its CTA reaches it.
struct PNode {
  CUtensorMap tmap;  // input tile map (tensor TMA), valid if use_tmap
  uint32_t box_bytes;
  int32_t use_tmap;
  int32_t in_stream;  // load the input evict-first (graph input; consumed intermediate of a tiled plan)
  DBuf in, out;
  int32_t op, scalar, tw, th;
  float T;
};
struct PCtrl {
  unsigned int done, epoch, ticket, pad1;  // ticket: next unclaimed ticket (dynamic mode)
};
struct PDep {
  int32_t sub;       // counter index (= sub-kernel id)
  uint32_t ntiles;   // its tiles per execute
};
struct PChunk {      // one discard ticket: lines [l0, l0 + n) of rect d (row-major, lpr per row)
  int32_t d;
  int32_t n;
  int64_t l0;
};
// Ticket descriptor: kind (4 bits: node id, or PK_DISCARD) | check (1) | group (19) |
// payload (40).  check = first ticket of its group in this CTA's list: the producer warp
// verifies the group's dependencies there (and only there).
// Tile payload: bz (12) | by (14) | bx (14); discard payload: chunk index.
constexpr uint64_t PK_DISCARD = 15, PK_STOP = 14, PK_CHECK = 1ull << 59;
constexpr int PGROUP_BITS = 19;
__host__ __device__ inline int ticket_group(uint64_t d) { return (int)((d >> 40) & ((1u << PGROUP_BITS) - 1)); }
__host__ __device__ inline uint64_t pack_ticket(uint64_t kind, uint64_t group, uint64_t payload) {
  return (kind << 60) | (group << 40) | payload;
}
__host__ __device__ inline uint64_t tile_payload(uint64_t bx, uint64_t by, uint64_t bz) {
  return (bz << 28) | (by << 14) | bx;
}
struct PParams {
  const PNode* nodes;
  const uint64_t* desc;     // [G][per_cta] tickets, STOP-padded
  int64_t per_cta;          // static: tickets per CTA list; dynamic: 0
  int64_t total;            // dynamic: tickets in the global order
  const int32_t* dep_off;   // CSR over groups
  const PDep* deps;
  const DRect* drects;
  const PChunk* chunks;
  int32_t nsub;             // groups < nsub are sub-kernels (counted); the rest discard lists
  int32_t pad;
  unsigned int* cnt;        // completion counters, one per sub-kernel
  PCtrl* ctrl;
  int64_t stage_bytes;      // one ring slot
  int32_t nslots;
  int32_t nnodes;
  TraceBuf tb;
};

__device__ __forceinline__ void nbar_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void mbar_arrive(uint64_t* m) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ktd::smem_u32(m)) : "memory");
}
__device__ __forceinline__ bool mbar_test(uint64_t* m, unsigned parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred P;\n mbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n selp.u32 %0, 1, 0, P;\n}"
      : "=r"(ok)
      : "r"(ktd::smem_u32(m)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void red_release_add(unsigned int* p, unsigned int v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
constexpr unsigned FULL = 0xFFFFFFFFu;

__device__ __forceinline__ ktd::Tile ticket_tile(const PNode& nd, uint64_t d) {
  const int bx = (int)(d & 0x3FFF), by = (int)((d >> 14) & 0x3FFF);
  ktd::Tile t;
  t.z = (int64_t)((d >> 28) & 0xFFF);
  t.x0 = (int64_t)nd.tw * bx;
  t.y0 = (int64_t)nd.th * by;
  t.x1 = min(t.x0 + nd.tw, nd.out.W);
  t.y1 = min(t.y0 + nd.th, nd.out.H);
  t.fw = nd.tw;
  t.pad = 0;
  return t;
}

// Producer warp: wait until every dependency group of `group` is complete this epoch.
// Polls are relaxed (no L1 invalidation per poll); one acquire once they are satisfied.
__device__ __forceinline__ unsigned int ld_relaxed(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void wait_group(const PParams& p, int group, unsigned epoch, int lane) {
  const int a = p.dep_off[group], b = p.dep_off[group + 1];
  for (int i = a + lane; i < b; i += 32) {
    const PDep dp = p.deps[i];
    const unsigned target = epoch * dp.ntiles;
    if ((int)(ld_relaxed(p.cnt + dp.sub) - target) < 0) {
      for (unsigned long long w = 0; (int)(ld_relaxed(p.cnt + dp.sub) - target) < 0;)
        kt_spin(w, 100, "PERSISTENT sub-kernel counter", dp.sub);
    }
    (void)ld_acquire(p.cnt + dp.sub);
  }
  __syncwarp();
}
// mbarrier wait that suspends between probes (off the compute warps' critical path)
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* m, unsigned parity) {
  asm volatile(
      "{\n .reg .pred P;\n KT_WS_%=:\n mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1, %2;\n @!P bra KT_WS_%=;\n}" ::"r"(
          ktd::smem_u32(m)),
      "r"(parity), "r"(1000000u)
      : "memory");
}

// Warp roles: NG compute groups of PCOMP_WARPS warps, one producer warp (dependency check
// + TMA issue into a ring of nslots staging slots shared by the groups), one publisher
// warp (publishes finished tiles to the sub-kernel counters with one gpu-scope release
// per run of consecutive tiles of the same sub-kernel).  Ticket k of the CTA uses slot
// k mod nslots and compute group k mod NG, so the groups share one pool of slots (a group
// busy with a long tile does not hold prefetch slots idle).  The compute warps free a
// slot themselves (s_empty), so neither a dependency poll nor a release fence ever sits
// between a finished tile and the refill of its slot.  The publisher reads finished
// tiles from its own queue (PUBQ entries, s_done barriers); the producer keeps at most
// PUBQ - PSTAGES_MAX tickets ahead of it, so a queue entry is never reused early.
constexpr int PUBQ = 64;
constexpr int DYN_B = 2;  // tickets per claim (dynamic mode)
template <int NG, int MINB>
__global__ void __launch_bounds__(NG * PCOMP_THREADS + 64, MINB) persistent_kernel(const __grid_constant__ PParams p) {
  __shared__ __align__(8) uint64_t s_full[PSTAGES_MAX];
  __shared__ __align__(8) uint64_t s_empty[PSTAGES_MAX];
  __shared__ __align__(8) uint64_t s_done[PUBQ];
  __shared__ uint64_t s_desc[PSTAGES_MAX];
  __shared__ ktd::Tile s_tile[PSTAGES_MAX];
  __shared__ int32_t s_pub[PUBQ];          // group of finished ticket k (k mod PUBQ)
  __shared__ int32_t s_pubk;  // tickets the publisher has consumed (shared atomics: a lock-free
                              // progress counter, written by the publisher, read by the producer)
  __shared__ __align__(64) PNode s_nodes[PMAX_NODES];
  __shared__ unsigned int s_epoch;
  __shared__ int32_t s_okg[64];
  extern __shared__ __align__(128) uint8_t ktsm[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int S = p.nslots;
  if (tid < 64) s_okg[tid] = -1;
  for (int i = tid; i < p.nnodes * (int)(sizeof(PNode) / 4); i += blockDim.x)
    reinterpret_cast<uint32_t*>(s_nodes)[i] = reinterpret_cast<const uint32_t*>(p.nodes)[i];
  if (tid == 0) {
    s_epoch = *(volatile unsigned int*)&p.ctrl->epoch;
    s_pubk = 0;
    for (int s = 0; s < S; ++s) {
      ktd::mbar_init(&s_full[s], 1);
      ktd::mbar_init(&s_empty[s], PCOMP_THREADS);
    }
    for (int q = 0; q < PUBQ; ++q) ktd::mbar_init(&s_done[q], PCOMP_THREADS);
    ktd::fence_proxy_async();
  }
  __syncthreads();
  const unsigned int epoch = s_epoch;
  const uint64_t* my = p.desc + (int64_t)blockIdx.x * p.per_cta;
  if (warp == NG * PCOMP_WARPS) {
    // ------------------------------ producer warp ------------------------------
    int s = 0, stops = 0;
    unsigned ph = 0;  // bit s: parity of slot s's current use
    uint64_t batch = 0;
    const bool dyn = p.per_cta == 0;
    // dynamic: chunks of DYN_B consecutive tickets claimed from the global counter; the
    // claim of the next chunk is issued when a chunk starts, so its latency overlaps it
    unsigned next = 0;
    if (dyn && lane == 0) next = atomicAdd(&p.ctrl->ticket, (unsigned)DYN_B);
    for (int64_t k = 0;; ++k) {
      if (dyn) {
        if ((k % DYN_B) == 0) {
          const unsigned base = __shfl_sync(FULL, next, 0);
          if (lane == 0 && base < p.total) next = atomicAdd(&p.ctrl->ticket, (unsigned)DYN_B);
          batch = lane < DYN_B && (int64_t)base + lane < p.total ? p.desc[base + lane] : pack_ticket(PK_STOP, 0, 0);
        }
      } else if ((k & 31) == 0) {
        batch = k + lane < p.per_cta ? my[k + lane] : pack_ticket(PK_STOP, 0, 0);
      }
      const uint64_t d = __shfl_sync(FULL, batch, dyn ? (int)(k % DYN_B) : (int)(k & 31));
      if (k >= S) ktd::mbar_wait(&s_empty[s], ((ph >> s) & 1u) ^ 1u);
      for (unsigned long long w = 0; (int)k - atomicAdd(&s_pubk, 0) > PUBQ - PSTAGES_MAX;)  // publisher queue bound
        kt_spin(w, 200, "PERSISTENT publisher queue", k);
      const uint64_t kind = d >> 60;
      if (kind == PK_STOP) {  // one STOP per compute group: tickets k .. k+NG-1
        if (lane == 0) {
          s_desc[s] = d;
          mbar_arrive(&s_full[s]);
        }
        __syncwarp();
        if (++stops == NG) break;
        ph ^= 1u << s;
        s = s + 1 == S ? 0 : s + 1;
        continue;
      }
      const uint64_t tq0 = p.tb.rec ? gtimer() : 0;
      if (d & PK_CHECK) {
        wait_group(p, ticket_group(d), epoch, lane);
      } else if (dyn) {  // dynamic: a small cache of groups already verified by this CTA
        const int gr = ticket_group(d);
        if (s_okg[gr & 63] != gr) {
          wait_group(p, gr, epoch, lane);
          if (lane == 0) s_okg[gr & 63] = gr;
          __syncwarp();
        }
      }
      if (lane == 0) {
        s_desc[s] = d;
        if (kind == PK_DISCARD) {
          mbar_arrive(&s_full[s]);
        } else {
          const PNode& nd = s_nodes[kind];
          const ktd::Tile t = ticket_tile(nd, d);
          s_tile[s] = t;
          if (nd.scalar) {
            mbar_arrive(&s_full[s]);
          } else {
            ktd::fence_proxy_async();
            ktd::stage_issue_tmap(nd.op, &p.nodes[kind].tmap, nd.box_bytes, nd.in, t, ktsm + s * p.stage_bytes,
                                  &s_full[s], nd.in_stream != 0);
          }
          if (p.tb.rec) trace_put(p.tb, d, 1, tq0, gtimer());
        }
      }
      __syncwarp();
      ph ^= 1u << s;
      s = s + 1 == S ? 0 : s + 1;
    }
  } else if (warp == NG * PCOMP_WARPS + 1) {
    // ------------------------------ publisher warp ------------------------------
    unsigned long long ph = 0;  // bit q: parity of queue entry q
    int cur = -1;               // sub-kernel of the pending run
    unsigned pend = 0;          // finished tiles not yet published
    int stops = 0;
    for (int k = 0;; ++k) {
      const int q = k & (PUBQ - 1);
      const unsigned par = (unsigned)(ph >> q) & 1u;
      if (pend && !mbar_test(&s_done[q], par)) {  // nothing more finished right now: publish
        if (lane == 0) red_release_add(p.cnt + cur, pend);
        pend = 0;
      }
      for (unsigned long long w = 0; !mbar_test(&s_done[q], par);) kt_spin(w, 64, "PERSISTENT finished tile", k);
      const int group = s_pub[q];
      __syncwarp();
      if (lane == 0) atomicExch(&s_pubk, k + 1);
      ph ^= 1ull << q;
      if (group < 0) {  // STOP of one compute group
        if (++stops == NG) break;
        continue;
      }
      if (group >= p.nsub) continue;  // discard chunk: nobody waits on it
      if (group != cur && pend) {
        if (lane == 0) red_release_add(p.cnt + cur, pend);
        pend = 0;
      }
      cur = group;
      ++pend;
    }
    if (pend && lane == 0) red_release_add(p.cnt + cur, pend);
  } else {
    // ------------------------------ compute groups ------------------------------
    const int cg = warp / PCOMP_WARPS, gtid = tid - cg * PCOMP_THREADS;
    for (int k = cg;; k += NG) {
      const int s = k % S;
      ktd::mbar_wait(&s_full[s], (unsigned)(k / S) & 1u);
      const uint64_t d = s_desc[s];
      const uint64_t kind = d >> 60;
      const int q = k & (PUBQ - 1);
      if (kind == PK_STOP) {
        if (gtid == 0) s_pub[q] = -1;
        mbar_arrive(&s_done[q]);
        break;
      }
      const uint64_t tc0 = p.tb.rec ? gtimer() : 0;
      if (kind == PK_DISCARD) {
        const PChunk c = p.chunks[d & 0xFFFFFFFFFFull];
        const DRect& r = p.drects[c.d];
        const int64_t h = r.y1 - r.y0;
        for (int64_t i = gtid; i < c.n; i += PCOMP_THREADS) {
          const int64_t j = c.l0 + i, row = j / r.lpr, l = j - row * r.lpr;
          const int64_t z = r.z0 + row / h, y = r.y0 + row % h;
          ktd::discard_line(r.base + drect_zoff(r, z) + y * r.pitch + r.lb0 + 128 * l);
        }
      } else {
        const PNode& nd = s_nodes[kind];
        const ktd::Tile t = s_tile[s];
        uint8_t* buf = ktsm + s * p.stage_bytes;
        if (nd.scalar) {
          ktd::scalar_tile(nd.op, nd.in, nd.out, t, nd.T, PCOMP_THREADS, gtid);
        } else {
          if ((nd.op == 1 || nd.op == 3) && ktd::needs_fix(nd.op, nd.in, t)) {
            ktd::stage_fix(nd.op, nd.in, t, buf, PCOMP_THREADS, gtid, 1 + NG + cg);
            nbar_sync(1 + cg, PCOMP_THREADS);
          }
          ktd::compute_tile(nd.op, nd.out, t, buf, nd.T, PCOMP_THREADS, gtid);
        }
        if (p.tb.rec && gtid == 0) trace_put(p.tb, d, 2, tc0, gtimer());
      }
      mbar_arrive(&s_empty[s]);  // this thread is done with the slot
      if (gtid == 0) s_pub[q] = ticket_group(d);
      // every compute thread arrives (release.cta) after its tile writes; the publisher
      // acquires the completed phase before its gpu-scope release (cumulative)
      mbar_arrive(&s_done[q]);
    }
  }
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    unsigned int old = atomicAdd(&p.ctrl->done, 1u);
    if (old == gridDim.x - 1) {
      p.ctrl->done = 0;
      p.ctrl->ticket = 0;
      __threadfence();
      atomicAdd(&p.ctrl->epoch, 1u);
    }
  }
}

// ------------------------------------------------------------------------------------
// footprint discovery (ktiler_discover_footprint): fill / perturb / compare kernels
// ------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t disc_hash(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return (uint32_t)(x ^ (x >> 31));
}
// byte i of a region = 1 + hash % 254 (never 0 or 255: a {0,255}-valued output always
// differs from the fill, so no written byte hides behind an equal fill value)
__global__ void disc_fill_kernel(uint8_t* p, int64_t n, uint64_t salt) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = (uint8_t)(1 + disc_hash(salt ^ ((uint64_t)i * 0x100000001B3ull)) % 254);
}
// bytes [a, b) of a region: XOR with a nonzero hash byte (every byte changes)
__global__ void disc_perturb_kernel(uint8_t* p, int64_t a, int64_t b, uint64_t salt) {
  for (int64_t i = a + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < b; i += (int64_t)gridDim.x * blockDim.x)
    p[i] ^= (uint8_t)(1 + disc_hash(salt ^ ((uint64_t)i * 0x100000001B3ull)) % 255);
}
// written |= (cur != snap)
__global__ void disc_diff_kernel(const uint8_t* cur, const uint8_t* snap, uint8_t* written, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    written[i] |= (uint8_t)(cur[i] != snap[i]);
}
// *flag |= any byte with written != 0 differs between cur and ref
__global__ void disc_cmp_kernel(const uint8_t* cur, const uint8_t* ref, const uint8_t* written, int64_t n,
                                unsigned int* flag) {
  unsigned int d = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    d |= (unsigned int)(written[i] && cur[i] != ref[i]);
  if (__syncthreads_or((int)d) && threadIdx.x == 0) atomicOr(flag, 1u);
}

// ------------------------------------------------------------------------------------

// ------------------------------------------------------------------------------------
// host side
// ------------------------------------------------------------------------------------
typedef void (*kfn_t)(KParams);
kfn_t deep_kernel(int op);

kfn_t vec_kernel(int op) {
  switch (op) {
    case 0: return op_kernel<0, false>;
    case 1: return op_kernel<1, false>;
    case 2: return op_kernel<2, false>;
    case 3: return op_kernel<3, false>;
    case 6: return op_kernel<6, false>;
    case 7: return op_kernel<7, false>;
    default: return op_kernel<4, false>;
  }
}
kfn_t vec_kernel_lean(int op, bool one) {  // one: a one-slot staging ring (one tile per CTA)
  switch (op) {
    case 0: return one ? op_kernel<0, false, 1, true> : op_kernel<0, false, 2, true>;
    case 1: return one ? op_kernel<1, false, 1, true> : op_kernel<1, false, 2, true>;
    case 2: return one ? op_kernel<2, false, 1, true> : op_kernel<2, false, 2, true>;
    case 3: return one ? op_kernel<3, false, 1, true> : op_kernel<3, false, 2, true>;
    case 4: return one ? op_kernel<4, false, 1, true> : op_kernel<4, false, 2, true>;
    case 6: return one ? op_kernel<6, false, 1, true> : op_kernel<6, false, 2, true>;
    case 7: return one ? op_kernel<7, false, 1, true> : op_kernel<7, false, 2, true>;
    default: return nullptr;
  }
}
kfn_t scalar_kernel(int op) {
  switch (op) {
    case 0: return op_kernel<0, true>;
    case 1: return op_kernel<1, true>;
    case 2: return op_kernel<2, true>;
    case 3: return op_kernel<3, true>;
    default: return op_kernel<4, true>;
  }
}

struct Launch {
  int node = -1;  // -1: discard-only
  kt::Node* n = nullptr;
  KParams kp;
  int64_t blocks = 0;
  dim3 block;
  int smem = 0;
  int64_t resident = 0;  // CTAs of this kernel that fit the device at once
  int64_t grid = 0;      // CTAs of the last prepared launch (prep_launch)
  int sub = -1;          // schedule sub-kernel (kernel launches) / discard list (DAG discards)
  std::vector<int32_t> crects;  // OP_CUSTOM rect list
  int cap_per_sm = 0;    // > 0: grid capped at this many CTAs per SM (grid-stride through the ring)
  bool one = false;      // one tile per CTA by construction (tiled GRAPH_DAG / WAVE): one-slot ring kernel
};

}  // namespace

struct ktiler_plan_s {
  kt::Graph g;
  kt::Schedule s;
  ktiler_fragment_policy pol{};
  double plan_ms = 0;
  std::vector<Launch> launches;
  std::vector<Launch> dag_disc;  // GRAPH_DAG: discard launches (sub = the discard list)
  int device = -1;
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  // persistent state
  void* dmem = nullptr;
  PParams pp{};
  int pctas = 0;
  int pminb = 2;
  int pgroups = 1;
  int pthreads = 0;
  int psmem = 0;
  void (*pfn)(PParams) = nullptr;
  int64_t skew = 0;
  bool has_custom = false;
  TraceBuf tb{nullptr, nullptr, 0};
  bool executed = false;
  ktiler_status sticky = KTILER_OK;  // a failed first-execute setup: the plan stays unusable
  // ring buffers (ktiler_buffer_desc.ring_frames): per sub-kernel, the earlier sub-kernels
  // that must finish first because they read (or write) the frame its writes overwrite
  std::vector<std::vector<int32_t>> war;
  // FLOW state (KTILER_EXEC_FLOW): roles (ktiler_plan_set_flow_roles; empty = automatic)
  std::vector<int32_t> flow_node_role, flow_slot_role;
  ktflow::FParams fp{};
  void (*ffn)(ktflow::FParams) = nullptr;
  int fctas = 0, fthreads = 0, fsmem = 0;
  void* fmem = nullptr;
  // ktiler_plan_attach_halo: the strip exchange run before the schedule in every execute
  ktiler_comm_t halo_comm = nullptr;
  int32_t halo_rank = 0, halo_rows = 0;
  // GRAPH_CHAIN state: one device block (epoch | flags | dcount | prefix) and the tail
  void* cmem = nullptr;
  std::vector<void*> hmem;  // halo-reader counters of consumer discards
  unsigned int* epoch = nullptr;
  std::vector<Launch> chain_tail;
  ~ktiler_plan_s() {
    if (exec) cudaGraphExecDestroy(exec);
    if (graph) cudaGraphDestroy(graph);
    if (dmem) cudaFree(dmem);
    if (fmem) cudaFree(fmem);
    if (tb.rec) cudaFree(tb.rec);
    if (cmem) cudaFree(cmem);
    for (void* m : hmem) cudaFree(m);
  }
};

namespace {
int dag_order_node();
bool dag_order_edges(const ktiler_plan_s* P);
}  // namespace
namespace {

using kt::fail;

DBuf dbuf(const kt::Buffer& b) {
  return DBuf{(uint8_t*)b.d.base, b.d.width, b.d.height, b.d.pitch_bytes, b.d.frame_stride_bytes,
              (int32_t)b.d.ring_frames, 0};
}

bool discardable(const kt::Buffer& b) { return (b.d.pitch_bytes % 128 == 0) && (b.d.frame_stride_bytes % 128 == 0); }

// With KTILER_PF_CONSUMER_DISCARD in a tiled plan, buffer b's lines are dropped by its only
// reader as soon as they are staged (A44): no discard list is needed for it.
bool consumer_drops(const ktiler_plan_s* P, int b) {
  const kt::Graph& g = P->g;
  if (!(P->pol.flags & KTILER_PF_CONSUMER_DISCARD) || P->s.nfrag <= 1) return false;
  const kt::Buffer& B = g.bufs[b];
  if (!(B.d.flags & KTILER_BUF_INTERNAL) || B.readers.size() != 1 || B.writer < 0) return false;
  const kt::Node& n = g.nodes[B.readers[0]];
  if (n.scalar || (n.op != KTILER_OP_DOWN2 && n.op != KTILER_OP_THRESH)) return false;
  const kt::Access& r = n.acc[n.racc];
  if (r.buf != b || r.hl || r.hr || r.ht || r.hb) return false;
  // consumer_discard drops only the lines wholly inside one block's input rect: the
  // reader's blocks cover every line only when a block's input row is a whole number of
  // lines (down2 reads 2 bytes, thresh 4 bytes per output pixel); otherwise the lines that
  // straddle two blocks still need the scheduled list
  const int64_t eb = n.op == KTILER_OP_DOWN2 ? 2 : 4;
  return (eb * n.acc[n.wacc].ax) % 128 == 0;
}

DRect drect(const kt::Graph& g, const kt::Discard& d) {
  const kt::Buffer& b = g.bufs[d.buf];
  DRect r;
  r.base = (uint8_t*)b.d.base;
  r.pitch = b.d.pitch_bytes;
  r.fstride = b.d.frame_stride_bytes;
  r.ring = (int32_t)b.d.ring_frames;
  r.pad = 0;
  r.lb0 = (d.xb0 + 127) & ~127ll;
  int64_t lb1 = d.xb1 & ~127ll;
  r.lpr = lb1 > r.lb0 ? (lb1 - r.lb0) / 128 : 0;
  r.y0 = d.y0; r.y1 = d.y1; r.z0 = d.z0; r.z1 = d.z1;
  return r;
}

// Ring buffers: frame z of a ring of R frames overwrites the slot of frame
// z - R, so every writer of frame z must follow every reader (and the writer) of frame
// z - R — write-after-read / write-after-write order the paper's RAW-only model
// does not have.  Per sub-kernel, the list of such earlier sub-kernels
// (P->war).  Total-order executors (STREAM, GRAPH) need them to precede it in the order
// (else KTILER_E_UNTILEABLE: a fragment spans R frames or more); GRAPH_DAG adds them as
// edges; the other executors do not support rings.
ktiler_status ring_analysis(ktiler_plan_s* P) {
  const kt::Graph& g = P->g;
  const kt::Schedule& S = P->s;
  const int nsub = (int)S.subs.size();
  P->war.assign(nsub, {});
  bool any = false;
  for (auto& b : g.bufs) any |= b.d.ring_frames > 0;
  if (!any) return KTILER_OK;
  const int m = P->pol.exec_mode;
  if (m != KTILER_EXEC_STREAM && m != KTILER_EXEC_GRAPH && m != KTILER_EXEC_GRAPH_DAG)
    return fail(KTILER_E_UNSUPPORTED, "ring buffers (ring_frames) need STREAM, GRAPH or GRAPH_DAG");
  for (int bi = 0; bi < (int)g.bufs.size(); ++bi) {
    const kt::Buffer& B = g.bufs[bi];
    const int64_t R = B.d.ring_frames, F = B.d.frames;
    if (!R) continue;
    std::vector<std::vector<int32_t>> users(F);  // per frame: sub-kernels reading or writing it
    std::vector<std::vector<int32_t>> writers(F);
    for (int si = 0; si < nsub; ++si) {
      const kt::SubKernel& sk = S.subs[si];
      const kt::Node& n = g.nodes[sk.node];
      bool rd = false, wr = false;
      for (auto& a : n.acc)
        if (a.buf == bi) (a.mode == KTILER_WRITE ? wr : rd) = true;
      if (!rd && !wr) continue;
      std::vector<uint8_t> seen(F, 0);
      for (auto& r : sk.rects)
        for (int64_t z = r.z0; z < r.z1; ++z) seen[z] = 1;
      for (int64_t z = 0; z < F; ++z)
        if (seen[z]) {
          users[z].push_back(si);
          if (wr) writers[z].push_back(si);
        }
    }
    for (int64_t z = R; z < F; ++z)
      for (int32_t w : writers[z])
        for (int32_t u : users[z - R]) {
          if (u == w) return fail(KTILER_E_UNTILEABLE, "ring buffer " + std::to_string(bi) + ": one sub-kernel spans frames " +
                                                           std::to_string(z - R) + " and " + std::to_string(z) + " of a " +
                                                           std::to_string(R) + "-frame ring");
          if (m != KTILER_EXEC_GRAPH_DAG && u > w)
            return fail(KTILER_E_UNTILEABLE, "ring buffer " + std::to_string(bi) + " of " + std::to_string(R) +
                                                 " frames: frame " + std::to_string(z) + " is written before frame " +
                                                 std::to_string(z - R) + " is read in this order (a fragment spans >= " +
                                                 std::to_string(R) + " frames): use a larger ring");
          if (u > w) return fail(KTILER_E_UNTILEABLE, "ring buffer: a reader of frame z-R follows the writer of z in the order");
          P->war[w].push_back(u);
        }
  }
  for (auto& v : P->war) {
    std::sort(v.begin(), v.end());
    v.erase(std::unique(v.begin(), v.end()), v.end());
  }
  return KTILER_OK;
}

// PF_PDL edge policy: an edge from launch `prod` is programmatic when several fragments
// overlap (nfrag > 1: GRAPH_DAG, profiles/r02_dag_pdl_sweep.txt) or when `prod` is a small
// launch of at most 2 CTAs per SM (a latency-bound chain of small kernels, where the
// consumer's early CTAs take idle SMs — HS 256^2 / 512^2 x 500 JI, 64 / 256 CTAs: 2.15 /
// 2.26 vs 2.39 / 2.50 ms, profiles/r02c_hs_pyramid.jsonl).  In a one-fragment plan larger
// producers lose (4096^2, 512-2048 CTAs: 52.5-54.5 vs 48-50 us; 64 x 8K untiled: 3.22 vs
// 3.19 ms).  STREAM launches are host-latency bound, so there every producer edge is
// programmatic (HS 1024^2 x 500: 3.86 vs 5.12 ms).  KTILER_PDL_ONE_FRAGMENT=1
// (experiment): every producer edge.
static bool pdl_edge(const ktiler_plan_s* P, const Launch& prod) {
  static const bool one = getenv("KTILER_PDL_ONE_FRAGMENT") && atoi(getenv("KTILER_PDL_ONE_FRAGMENT")) != 0;
  if (!(P->pol.flags & KTILER_PF_PDL) || prod.node < 0 || prod.n->op == KTILER_OP_CUSTOM) return false;
  if (P->s.nfrag > 1 || one || P->pol.exec_mode == KTILER_EXEC_STREAM) return true;
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, P->device);
  return prod.grid > 0 && prod.grid <= 2 * (int64_t)std::max(nsm, 1);
}

void build_launches(ktiler_plan_s* P) {
  const kt::Graph& g = P->g;
  const bool disc = (P->pol.flags & KTILER_PF_DISCARD_DEAD) != 0;
  // griddepcontrol in the kernels is a no-op on a launch without programmatic producers
  const bool pdl = (P->pol.flags & KTILER_PF_PDL) != 0;
  // GRAPH_DAG and GRAPH_CHAIN keep each sub-kernel's discard list apart (dag_disc, sub =
  // the list's sub-kernel): DAG makes them graph nodes, CHAIN attaches them to later launches
  const bool dag = P->pol.exec_mode == KTILER_EXEC_GRAPH_DAG || P->pol.exec_mode == KTILER_EXEC_GRAPH_CHAIN ||
                   P->pol.exec_mode == KTILER_EXEC_GRAPH_WAVE;
  std::vector<DRect> pending;
  auto flush_disc_only = [&](size_t keep) {
    while (pending.size() > keep) {
      Launch L;
      std::memset(&L.kp, 0, sizeof(L.kp));
      L.kp.pdl = pdl;
      size_t n = std::min<size_t>(MAXD, pending.size());
      L.kp.ndisc = (int32_t)n;
      L.kp.dpre[0] = 0;
      for (size_t i = 0; i < n; ++i) {
        L.kp.d[i] = pending[i];
        L.kp.dpre[i + 1] = L.kp.dpre[i] + L.kp.d[i].lpr * (int64_t)(pending[i].y1 - pending[i].y0) * (pending[i].z1 - pending[i].z0);
      }
      pending.erase(pending.begin(), pending.begin() + n);
      int64_t lines = L.kp.dpre[n];
      L.blocks = std::max<int64_t>(1, std::min<int64_t>(1184, (lines + 255) / 256));
      L.block = dim3(256);
      P->launches.push_back(L);
    }
  };
  for (size_t si = 0; si < P->s.subs.size(); ++si) {
    const kt::SubKernel& sk = P->s.subs[si];
    const kt::Node& n = g.nodes[sk.node];
    if (n.op == KTILER_OP_CUSTOM) {
      flush_disc_only(0);
      Launch L;
      L.node = sk.node;
      L.n = const_cast<kt::Node*>(&n);
      L.sub = (int)si;  // GRAPH_DAG adds launches by sub-kernel
      for (auto& r : sk.rects) {
        int32_t v[6] = {r.x0, r.y0, r.z0, r.x1, r.y1, r.z1};
        L.crects.insert(L.crects.end(), v, v + 6);
      }
      P->launches.push_back(L);
    } else {
      const kt::Access& w = n.acc[n.wacc];
      const kt::Access& r = n.acc[n.racc];
      for (size_t c = 0; c < sk.rects.size(); c += MAXR) {
        if (pending.size() > (size_t)MAXD) flush_disc_only(MAXD);
        Launch L;
        std::memset(&L.kp, 0, sizeof(L.kp));
        L.node = sk.node;
        L.n = const_cast<kt::Node*>(&n);
        L.kp.in = dbuf(g.bufs[r.buf]);
        L.kp.out = dbuf(g.bufs[w.buf]);
        if (n.racc2 >= 0) L.kp.aux = dbuf(g.bufs[n.acc[n.racc2].buf]);
        // Staged reads with an L2 evict-first hint: graph inputs always (read once); in a
        // tiled plan also the intermediates read by one node only (that node is their last
        // reader), so a consumed line becomes the first eviction candidate and the dead
        // lines of earlier fragments stop crowding out the live ones (64 x 8K: 3.43 ->
        // 3.28 ms, A42).  Untiled plans keep the default policy (halo rows are
        // re-read by the next tile row much later).  KTILER_EVICT_READS=0/1 forces it.
        static const int evict_env = getenv("KTILER_EVICT_READS") ? atoi(getenv("KTILER_EVICT_READS")) : -1;
        const bool evict_reads = evict_env >= 0 ? evict_env != 0 : (P->s.nfrag > 1 && g.bufs[r.buf].readers.size() == 1);
        L.kp.in_stream = evict_reads || !g.written_by_node(r.buf);
        // consumer-side discard (PF_CONSUMER_DISCARD, A44): tiled plan, internal input with
        // this node as its only reader, read without halo, line-aligned rows
        const kt::Buffer& ib = g.bufs[r.buf];
        L.kp.cdisc = (P->pol.flags & KTILER_PF_CONSUMER_DISCARD) && P->s.nfrag > 1 && !n.scalar &&
                     (n.op == KTILER_OP_DOWN2 || n.op == KTILER_OP_THRESH) && (ib.d.flags & KTILER_BUF_INTERNAL) &&
                     ib.readers.size() == 1 && !r.hl && !r.hr && !r.ht && !r.hb && discardable(ib) &&
                     g.written_by_node(r.buf);
        L.kp.tw = (int32_t)w.ax;
        L.kp.th = (int32_t)w.ay;
        L.kp.T = n.T;
        L.kp.radius = n.radius;
        for (int k = 0; k <= 2 * n.radius && k < 2 * ktd::GAUSS_H + 1; ++k) L.kp.taps[k] = n.taps[k];
        // KTILER_PDL_TRIGGER=exit (experiment): dependents scheduled only as CTAs exit
        static const bool trig_exit = getenv("KTILER_PDL_TRIGGER") && !strcmp(getenv("KTILER_PDL_TRIGGER"), "exit");
        L.kp.pdl = pdl ? (trig_exit ? 2 : 1) : 0;
        if (!trig_exit && dag_order_edges(P) && g.in_ch[sk.node].empty() && !g.bufs[w.buf].d.ring_frames && sk.frag > 0)
          L.kp.pdl = 3;  // dispatch-order edge only: no producer to wait for
        size_t m = std::min<size_t>(MAXR, sk.rects.size() - c);
        L.kp.nrect = (int32_t)m;
        L.kp.rpre[0] = 0;
        for (size_t i = 0; i < m; ++i) {
          const kt::Rect6& q = sk.rects[c + i];
          L.kp.r[i] = {q.x0, q.y0, q.z0, q.x1, q.y1, q.z1};
          L.kp.rpre[i + 1] = L.kp.rpre[i] + q.count();
        }
        L.blocks = L.kp.rpre[m];
        L.sub = (int)si;
        if (!dag && c == 0 && !pending.empty()) {
          size_t nd = std::min<size_t>(MAXD, pending.size());
          L.kp.ndisc = (int32_t)nd;
          L.kp.dpre[0] = 0;
          for (size_t i = 0; i < nd; ++i) {
            L.kp.d[i] = pending[i];
            L.kp.dpre[i + 1] = L.kp.dpre[i] + pending[i].lpr * (int64_t)(pending[i].y1 - pending[i].y0) * (pending[i].z1 - pending[i].z0);
          }
          pending.erase(pending.begin(), pending.begin() + nd);
        }
        L.block = dim3(n.block[0], n.block[1], n.block[2]);
        L.kp.stage_bytes = n.scalar ? 0 : (ktd::stage_bytes(n.op, (int)w.ax, (int)w.ay) + 127) & ~127;
        L.kp.nstage = 2;
        L.smem = (int)(2 * L.kp.stage_bytes);
        // KTILER_STAGES=S (experiment): sub-kernels of a tiled plan whose input is
        // an intermediate (L2-resident) run one resident wave of CTAs that grid-stride over
        // their tiles through an S-deep staging ring instead of one tile per CTA
        static const int stages_env = getenv("KTILER_STAGES") ? atoi(getenv("KTILER_STAGES")) : 0;
        if (stages_env > 2 && !n.scalar && P->s.nfrag > 1 && deep_kernel(n.op) && g.written_by_node(r.buf)) {
          L.kp.nstage = std::min(stages_env, KMAXST);
          L.smem = (int)(L.kp.nstage * L.kp.stage_bytes);
        }
        // KTILER_SRC_CTAS=K (experiment): the sub-kernels of a tiled plan that read a graph
        // input (the HBM-streaming source node) run at most K CTAs per SM, grid-striding through
        // a KTILER_SRC_STAGES-deep ring (default 3), so they stream without filling every SM
        // slot ahead of the previous fragment's consumer sub-kernels
        static const int src_ctas = getenv("KTILER_SRC_CTAS") ? atoi(getenv("KTILER_SRC_CTAS")) : 0;
        static const int src_stages = getenv("KTILER_SRC_STAGES") ? atoi(getenv("KTILER_SRC_STAGES")) : 3;
        if (src_ctas > 0 && !n.scalar && P->s.nfrag > 1 && !g.written_by_node(r.buf) &&
            (src_stages <= 2 || deep_kernel(n.op))) {
          L.kp.nstage = std::max(2, std::min(src_stages, KMAXST));
          L.smem = (int)(L.kp.nstage * L.kp.stage_bytes);
          L.cap_per_sm = src_ctas;
        }
        // tiled GRAPH_DAG / WAVE launches run one tile per CTA (prep_launch) unless overridden
        static const bool tpc_set = getenv("KTILER_TILES_PER_CTA") != nullptr;
        L.one = !tpc_set && L.kp.nstage <= 2 && L.cap_per_sm == 0 && P->s.nfrag > 1 &&
                (P->pol.exec_mode == KTILER_EXEC_GRAPH_DAG || P->pol.exec_mode == KTILER_EXEC_GRAPH_WAVE);
        P->launches.push_back(L);
      }
    }
    if (disc)
      for (auto& d : P->s.discards[si]) {
        if (!discardable(g.bufs[d.buf]) || consumer_drops(P, d.buf)) continue;  // A44: its reader drops it
        DRect dr = drect(g, d);
        if (dr.lpr > 0) pending.push_back(dr);
      }
    if (dag && !pending.empty()) {  // one discard node per list (chunks of MAXD rects)
      const size_t base = P->launches.size();
      flush_disc_only(0);
      for (size_t k = base; k < P->launches.size(); ++k) {
        P->launches[k].sub = (int)si;
        P->dag_disc.push_back(P->launches[k]);
      }
      P->launches.resize(base);
    }
  }
  flush_disc_only(0);
}

// GRAPH_DAG edges at sub-kernel level: exact sub-kernel dependencies (Schedule::sub_deps),
// the previous sub-kernel of the same node, and the run-ahead window (a sub-kernel with no
// producers in fragment f waits for the leaf sub-kernels of fragment f - window).
// Dispatch-order edges (GRAPH_DAG with PDL): the source sub-kernels of fragment f (nodes
// that read only graph inputs) get a programmatic edge from the sub-kernels of fragment
// f - 1 of the source's direct consumers, and skip griddepcontrol.wait (there is no
// producer data to wait for): fragment f's source is launched once fragment f - 1's first
// consumer has had all its CTAs dispatched (64 x 8K: 2.941 -> 2.920 ms).
// KTILER_DAG_ORDER_NODE (experiment): -1 / unset = that default, -2 = off, v >= 0 = edges
// from node v's sub-kernel instead (deeper nodes measured much slower).
int dag_order_node() {
  static const int v = getenv("KTILER_DAG_ORDER_NODE") ? atoi(getenv("KTILER_DAG_ORDER_NODE")) : -1;
  return v;
}
bool dag_order_edges(const ktiler_plan_s* P) {
  return (P->pol.flags & KTILER_PF_PDL) && P->pol.exec_mode == KTILER_EXEC_GRAPH_DAG && dag_order_node() != -2;
}

int dag_prio_mode() {
  static const int v = getenv("KTILER_DAG_PRIO") ? atoi(getenv("KTILER_DAG_PRIO")) : 0;
  return v;
}

std::vector<std::vector<int>> dag_edges(const ktiler_plan_s* P) {
  const kt::Schedule& S = P->s;
  const kt::Graph& g = P->g;
  const int nsub = (int)S.subs.size();
  const int window = P->pol.window > 0 ? P->pol.window : 2;
  if (P->pol.exec_mode == KTILER_EXEC_GRAPH_WAVE) {
    // wave(sub) = fragment + node depth; every sub-kernel of wave w depends on every
    // sub-kernel of the previous non-empty wave (a barrier).  Producers sit at a smaller
    // depth in the same or an earlier fragment, hence in an earlier wave.
    std::vector<int> depth(g.nodes.size(), 0);
    for (int v : g.topo)
      for (auto& c : g.in_ch[v]) depth[v] = std::max(depth[v], depth[c.u] + 1);
    int dmax = 0;
    for (int d : depth) dmax = std::max(dmax, d);
    std::vector<std::vector<int>> waves(S.nfrag + dmax + 1);
    for (int i = 0; i < nsub; ++i) waves[S.subs[i].frag + depth[S.subs[i].node]].push_back(i);
    std::vector<std::vector<int>> e(nsub);
    const std::vector<int>* prev = nullptr;
    for (auto& w : waves) {
      if (w.empty()) continue;
      if (prev)
        for (int i : w) e[i] = *prev;
      prev = &w;
    }
    return e;
  }
  std::vector<std::vector<int>> leaf_subs(S.nfrag), e(nsub);
  // leaf = no consumer inside the sub-kernel's cluster (Alg. 1 partitions; else the graph)
  std::vector<std::vector<uint8_t>> member(S.clusters.size(), std::vector<uint8_t>(g.nodes.size(), 0));
  for (size_t c = 0; c < S.clusters.size(); ++c)
    for (int v : S.clusters[c]) member[c][v] = 1;
  for (int i = 0; i < nsub; ++i) {
    const int v = S.subs[i].node, c = S.subs[i].cluster;
    bool leaf = true;
    for (const kt::Chan& ch : g.out_ch[v]) leaf = leaf && !(c < (int)member.size() && member[c][ch.v]);
    if (leaf) leaf_subs[S.subs[i].frag].push_back(i);
  }
  std::vector<int> last_of_node(g.nodes.size(), -1);
  for (int i = 0; i < nsub; ++i) {
    e[i].assign(S.sub_deps[i].begin(), S.sub_deps[i].end());
    if (i < (int)P->war.size()) e[i].insert(e[i].end(), P->war[i].begin(), P->war[i].end());  // ring WAR order
    const int prev = last_of_node[S.subs[i].node];
    if (prev >= 0) e[i].push_back(prev);
    const int f = S.subs[i].frag;
    if (S.sub_deps[i].empty() && f >= window) e[i].insert(e[i].end(), leaf_subs[f - window].begin(), leaf_subs[f - window].end());
    std::sort(e[i].begin(), e[i].end());
    e[i].erase(std::unique(e[i].begin(), e[i].end()), e[i].end());
    last_of_node[S.subs[i].node] = i;
  }
  return e;
}

// GRAPH_DAG: each discard list rides in the prologue of the earliest later launch that
// (transitively) follows every reader of the list's lines — usually the very next
// sub-kernel of the schedule — so dead lines leave L2 as early as in the linear graph,
// without extra graph nodes.  Lists with no such launch stay in dag_disc as nodes.
void fold_dag_discards(ktiler_plan_s* P) {
  const kt::Schedule& S = P->s;
  const int nsub = (int)S.subs.size();
  const std::vector<std::vector<int>> e = dag_edges(P);
  // ancestor bitsets in schedule order (every edge points to an earlier sub-kernel)
  const int words = (nsub + 63) / 64;
  std::vector<uint64_t> anc((size_t)nsub * words, 0);
  for (int i = 0; i < nsub; ++i) {
    uint64_t* a = &anc[(size_t)i * words];
    for (int d : e[i]) {
      const uint64_t* b = &anc[(size_t)d * words];
      for (int w = 0; w < words; ++w) a[w] |= b[w];
      a[d >> 6] |= 1ull << (d & 63);
    }
  }
  std::vector<int64_t> first_launch(nsub, -1);
  for (size_t k = 0; k < P->launches.size(); ++k) {
    const Launch& L = P->launches[k];
    if (L.node >= 0 && L.sub >= 0 && first_launch[L.sub] < 0) first_launch[L.sub] = (int64_t)k;
  }
  std::vector<Launch> rest;
  for (auto& D : P->dag_disc) {
    const std::vector<int32_t>& readers = S.discard_readers[D.sub];
    bool placed = false;
    for (int j = D.sub + 1; j < nsub && !placed; ++j) {
      if (first_launch[j] < 0) continue;
      const uint64_t* a = &anc[(size_t)j * words];
      bool ok = true;
      for (int r : readers) ok = ok && ((a[r >> 6] >> (r & 63)) & 1) != 0;
      if (!ok) continue;
      KParams& k = P->launches[first_launch[j]].kp;
      if (k.ndisc + D.kp.ndisc > MAXD) continue;
      for (int q = 0; q < D.kp.ndisc; ++q) {
        k.d[k.ndisc] = D.kp.d[q];
        k.dpre[k.ndisc + 1] = k.dpre[k.ndisc] + (D.kp.dpre[q + 1] - D.kp.dpre[q]);
        ++k.ndisc;
      }
      placed = true;
    }
    if (!placed) rest.push_back(D);
  }
  P->dag_disc.swap(rest);
}

// ---- tensor maps for TMA staging (driver entry point, resolved at first execute) ----
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
// L2 sector promotion of the TMA requests (KTILER_TMA_PROMOTION = 0 / 64 / 128 / 256 bytes;
// default 128: the DAG + PDL step 0.6-0.8% faster than with 256, 0 the same,
// profiles/r02c_policy_sweep.txt).
CUtensorMapL2promotion l2_promotion() {
  static const int v = getenv("KTILER_TMA_PROMOTION") ? atoi(getenv("KTILER_TMA_PROMOTION")) : 128;
  return v == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE
                : (v == 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                           : (v == 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B : CU_TENSOR_MAP_L2_PROMOTION_L2_256B));
}

EncodeTiledFn get_encode() {
  static EncodeTiledFn fn = nullptr;
  static bool tried = false;
  if (!tried) {
    tried = true;
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeTiledFn)f;
  }
  return fn;
}

// Input-tile map of built-in node n: the input buffer as 4-byte elements
// [frames][height][ceil(row bytes / 4)], box = the staged window of one full tile
// (ktd::stage_geo / stage_bytes).  False -> the kernels use per-row bulk copies instead.
bool make_tmap(const kt::Graph& g, const kt::Node& n, CUtensorMap* m, uint32_t* box_bytes) {
  if (getenv("KTILER_NO_TMAP")) return false;
  EncodeTiledFn enc = get_encode();
  if (!enc) return false;
  const kt::Access& w = n.acc[n.wacc];
  const kt::Buffer& B = g.bufs[n.acc[n.racc].buf];
  const int tw = (int)w.ax, th = (int)w.ay, nseg = (tw + 15) / 16;
  int bw = 0, bh = 0;  // box bytes per row, box rows
  switch (n.op) {
    case KTILER_OP_GRAY: bw = 48 * nseg; bh = th; break;
    case KTILER_OP_BLUR5: bw = 16 * (nseg + 2); bh = th + 4; break;
    case KTILER_OP_DOWN2: bw = 32 * nseg; bh = 2 * th; break;
    case KTILER_OP_SOBEL3: bw = 16 * (nseg + 2); bh = th + 2; break;
    case KTILER_OP_JACOBI: bw = 4 * (tw + 8); bh = th + 2; break;
    case KTILER_OP_GAUSS_F32: bw = 4 * (tw + 2 * ktd::GAUSS_H); bh = th + 2 * ktd::GAUSS_H; break;
    default: bw = 64 * nseg; bh = th; break;
  }
  const int window = ktd::stage_bytes(n.op, tw, th);
  if (bw % 16 || bw / 4 > 256 || bh > 256 || bw * bh != window) return false;
  if (B.d.pitch_bytes % 16 || B.d.frame_stride_bytes % 16) return false;
  const int64_t rowbytes = B.d.width * B.d.elem_bytes;
  cuuint64_t dims[3] = {(cuuint64_t)((rowbytes + 3) / 4), (cuuint64_t)B.d.height,
                        (cuuint64_t)(B.d.ring_frames ? B.d.ring_frames : B.d.frames)};
  cuuint64_t strides[2] = {(cuuint64_t)B.d.pitch_bytes, (cuuint64_t)B.d.frame_stride_bytes};
  cuuint32_t box[3] = {(cuuint32_t)(bw / 4), (cuuint32_t)bh, 1}, es[3] = {1, 1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 3, B.d.base, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, l2_promotion(), CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return false;
  *box_bytes = (uint32_t)(bw * bh);
  return true;
}

ktiler_status cuda_fail(cudaError_t e, const char* what) {
  return fail(KTILER_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

kfn_t deep_kernel(int op) {  // runtime ring depth (KParams::nstage > 2)
  switch (op) {
    case 0: return op_kernel<0, false, 0>;
    case 2: return op_kernel<2, false, 0>;
    case 3: return op_kernel<3, false, 0>;
    case 4: return op_kernel<4, false, 0>;
    default: return nullptr;
  }
}
kfn_t launch_fn(const Launch& L) {
  // KTILER_LEAN (experiment knob): 0 = full kernels, 1 = lean two-slot only, unset = lean, and
  // one-slot where the launch runs one tile per CTA (L.one, GRAPH_DAG / WAVE tiled plans)
  static const int lean_env = getenv("KTILER_LEAN") ? atoi(getenv("KTILER_LEAN")) : 2;
  if (lean_env && L.node >= 0 && !L.n->scalar && L.kp.nstage <= 2 && !L.kp.chain && !L.kp.hcnt && !L.kp.tb.rec &&
      L.kp.use_tmap && !L.kp.ndisc && vec_kernel_lean(L.n->op, false))
    return vec_kernel_lean(L.n->op, lean_env == 2 && L.one);
  if (L.node >= 0 && !L.n->scalar && L.kp.nstage > 2 && deep_kernel(L.n->op)) return deep_kernel(L.n->op);
  return L.node < 0 ? (kfn_t)discard_kernel : (L.n->scalar ? scalar_kernel(L.n->op) : vec_kernel(L.n->op));
}

// Dynamic-smem attribute + grid of one launch: the vector kernels grid-stride over their
// tiles with as many CTAs as fit the device at once.
ktiler_status prep_launch(ktiler_plan_s* P, Launch& L, kfn_t fn, int64_t* grid_out) {
  // static + dynamic may pass the 48 KB default.  The attribute is a per-function MAXIMUM
  // (occupancy follows each launch's own size), so it is raised once to the device's
  // opt-in limit: launches of one kernel with different ring depths never undercut it
  if (L.resident == 0) {
    cudaFuncAttributes fa{};
    cudaFuncGetAttributes(&fa, (const void*)fn);
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, P->device);
    const int want = optin - (int)fa.sharedSizeBytes;
    if (fa.maxDynamicSharedSizeBytes < want) {
      cudaError_t ea = cudaFuncSetAttribute((const void*)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, want);
      if (ea != cudaSuccess) return cuda_fail(ea, "cudaFuncSetAttribute (dynamic smem)");
    }
  }
  if (L.resident == 0) {
    int nsm = 0, occ = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, P->device);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, (int)(L.block.x * L.block.y * L.block.z), L.smem);
    L.resident = (int64_t)std::max(1, nsm) * std::max(1, occ);
  }
  int64_t grid = std::max<int64_t>(L.blocks, 1);
  if (L.cap_per_sm > 0) {  // KTILER_SRC_CTAS: K CTAs per SM grid-striding through the ring
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, P->device);
    *grid_out = std::min<int64_t>({grid, L.resident, (int64_t)L.cap_per_sm * std::max(1, nsm)});
    return KTILER_OK;
  }
  // deep staging ring (KTILER_STAGES, set at plan time): one resident wave of CTAs that
  // grid-stride over the sub-kernel's tiles
  if (L.kp.nstage > 2) {
    *grid_out = std::min<int64_t>(grid, L.resident);
    return KTILER_OK;
  }
  // grid-stride CTAs (x tiles_per_cta) in stream/graph modes; in GRAPH_DAG one CTA per
  // tile by default, so concurrent sub-kernels interleave at tile granularity
  static const int tpc_env = getenv("KTILER_TILES_PER_CTA") ? atoi(getenv("KTILER_TILES_PER_CTA")) : -1;
  const bool chain = P->pol.exec_mode == KTILER_EXEC_GRAPH_CHAIN;
  // Default: a launch much larger than the device (the untiled kernels) gets 2 tiles per
  // CTA and leaves the balancing to the hardware scheduler; smaller ones (sub-kernels) get
  // one resident wave of CTAs that grid-stride over the tiles (fewer CTA setups, no
  // partial last wave).  GRAPH_CHAIN: one tile per CTA (fine-grained flags).  GRAPH_DAG /
  // GRAPH_WAVE: one tile per CTA, so the hardware scheduler balances concurrent
  // sub-kernels tile by tile (64 x 8K, 0.5 x L2 resident budget: 4.03 ms vs 4.23 ms
  // grid-stride).  Measured on 64 x 8K; KTILER_TILES_PER_CTA overrides.
  // (a one-fragment plan has no concurrent sub-kernels: it is the untiled schedule and
  // takes the GRAPH rule, so the two replay identical launches)
  const bool concurrent =
      (P->pol.exec_mode == KTILER_EXEC_GRAPH_DAG || P->pol.exec_mode == KTILER_EXEC_GRAPH_WAVE) && P->s.nfrag > 1;
  int tpc = tpc_env >= 0 ? tpc_env : (L.blocks > 8 * L.resident ? 2 : ((chain || concurrent) ? 1 : 0));
  if (tpc_env < 0 && tpc == 2 && L.node >= 0 && !L.n->scalar && L.kp.stage_bytes && L.smem == (int)(2 * L.kp.stage_bytes)) {
    // double buffering halves the CTAs that fit by shared memory; when registers would
    // allow >= 1.5x as many single-buffer CTAs, the extra warps hide more latency than the
    // second buffer does (blur5: 0.97 -> 0.87 ms on 64 x 8K)
    int occ1 = 0, occ2 = 0;
    const int thr = (int)(L.block.x * L.block.y * L.block.z);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ1, fn, thr, (int)L.kp.stage_bytes);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, fn, thr, L.smem);
    if (2 * occ1 >= 3 * occ2) tpc = 1;
  }
  // a single staging buffer holds one tile: such a launch must not grid-stride
  if (L.node >= 0 && !L.n->scalar && L.kp.stage_bytes && L.smem < (int)(2 * L.kp.stage_bytes) && tpc != 1) tpc = 1;
  if (L.node >= 0 && !L.n->scalar) {
    if (tpc > 0) grid = (grid + tpc - 1) / tpc;
    else grid = std::min<int64_t>(grid, L.resident);
  }
  if (L.node >= 0 && !L.n->scalar && grid >= L.blocks && L.smem != (int)L.kp.stage_bytes) {
    // one tile per CTA: the second staging buffer is never used -> more resident CTAs
    L.smem = (int)L.kp.stage_bytes;
    L.resident = 0;
    return prep_launch(P, L, fn, grid_out);
  }
  // The launch's own CTAs share its discard lines (grid-stride): enlarging the grid for
  // them would turn multi-tile CTAs into one- or zero-tile CTAs that pay the CTA setup.
  // Discard-only launches size their grid to the lines.
  if (L.node < 0 && L.kp.ndisc) grid = std::max<int64_t>(1, std::min<int64_t>(1184, (L.kp.dpre[L.kp.ndisc] + 255) / 256));
  (void)chain;
  *grid_out = grid;
  return KTILER_OK;
}

// GRAPH_DAG: the sub-kernels as graph nodes whose edges are their exact dependencies
// (Schedule::sub_deps), the previous sub-kernel of the same kernel (keeps each kernel's
// order), and a run-ahead window — a source sub-kernel of fragment f waits for the leaf
// sub-kernels of fragment f - window — so at most `window` fragments are in flight (the
// L2 footprint stays bounded) while their launches overlap each other's gaps and tails.
// A discard node waits for every sub-kernel that reads the blocks it retires.
ktiler_status build_dag(ktiler_plan_s* P, cudaGraph_t* out) {
  const kt::Schedule& S = P->s;
  const kt::Graph& g = P->g;
  const int nsub = (int)S.subs.size();
  const int window = P->pol.window > 0 ? P->pol.window : 2;
  cudaGraph_t gr = nullptr;
  cudaError_t e = cudaGraphCreate(&gr, 0);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGraphCreate");
  std::vector<std::vector<cudaGraphNode_t>> nodes_of(nsub);
  const std::vector<std::vector<int>> edges = dag_edges(P);
  // PF_PDL: the edges from a sub-kernel's producers (Schedule::sub_deps; with
  // KTILER_DAG_PDL_EDGES=all every kernel edge) are programmatic: the consumer's CTAs may
  // become resident while the producer's last wave drains and wait in griddepcontrol.wait
  // (full completion + memory flush of every programmatic producer) before reading.
  const bool pdl = (P->pol.flags & KTILER_PF_PDL) != 0;
  static const bool pdl_all = getenv("KTILER_DAG_PDL_EDGES") && !strcmp(getenv("KTILER_DAG_PDL_EDGES"), "all");
  // KTILER_DAG_PDL_EDGES=chain (experiment): also the edge from the previous sub-kernel of
  // the same node (not the window edges)
  static const bool pdl_chain = getenv("KTILER_DAG_PDL_EDGES") && !strcmp(getenv("KTILER_DAG_PDL_EDGES"), "chain");
  // KTILER_DAG_PDL_EDGES=window (experiment): also the run-ahead window edges
  static const bool pdl_window = getenv("KTILER_DAG_PDL_EDGES") && !strcmp(getenv("KTILER_DAG_PDL_EDGES"), "window");
  auto add_node = [&](Launch& L, const std::vector<cudaGraphNode_t>& deps, const std::vector<uint8_t>& prog,
                      cudaGraphNode_t* node) -> ktiler_status {
    if (L.node >= 0 && L.n->op == KTILER_OP_CUSTOM) {
      // a user kernel (KTILER_OP_CUSTOM): its launch callback, stream-captured once for this
      // sub-kernel's rect list, becomes a child graph node with the same dependency edges
      cudaStream_t cs;
      cudaError_t ce = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
      if (ce != cudaSuccess) return cuda_fail(ce, "cudaStreamCreate");
      if ((ce = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal)) != cudaSuccess) {
        cudaStreamDestroy(cs);
        return cuda_fail(ce, "cudaStreamBeginCapture (custom)");
      }
      L.n->launch(L.n->user, L.crects.data(), (int32_t)(L.crects.size() / 6), (void*)cs);
      cudaGraph_t cg = nullptr;
      ce = cudaStreamEndCapture(cs, &cg);
      cudaStreamDestroy(cs);
      if (ce != cudaSuccess) return cuda_fail(ce, "cudaStreamEndCapture (custom launch callback)");
      ce = cudaGraphAddChildGraphNode(node, gr, deps.data(), deps.size(), cg);
      cudaGraphDestroy(cg);
      if (ce != cudaSuccess) return cuda_fail(ce, "cudaGraphAddChildGraphNode (custom)");
      return KTILER_OK;
    }
    kfn_t fn = launch_fn(L);
    int64_t grid = 0;
    ktiler_status ps = prep_launch(P, L, fn, &grid);
    if (ps) return ps;
    L.grid = grid;
    void* args[1] = {&L.kp};
    cudaKernelNodeParams kp = {};
    kp.func = (void*)fn;
    kp.gridDim = dim3((unsigned)grid);
    kp.blockDim = L.block;
    kp.sharedMemBytes = (unsigned)L.smem;
    kp.kernelParams = args;
    if (!pdl) {
      cudaError_t ee = cudaGraphAddKernelNode(node, gr, deps.data(), deps.size(), &kp);
      if (ee != cudaSuccess) return cuda_fail(ee, "cudaGraphAddKernelNode");
      return KTILER_OK;
    }
    cudaError_t ee = cudaGraphAddKernelNode(node, gr, nullptr, 0, &kp);
    if (ee != cudaSuccess) return cuda_fail(ee, "cudaGraphAddKernelNode");
    std::vector<cudaGraphEdgeData> ed(deps.size());
    for (size_t j = 0; j < deps.size(); ++j) {
      std::memset(&ed[j], 0, sizeof(ed[j]));
      if (!prog.empty() && prog[j]) {
        ed[j].from_port = cudaGraphKernelNodePortProgrammatic;
        ed[j].type = cudaGraphDependencyTypeProgrammatic;
      }
    }
    std::vector<cudaGraphNode_t> to(deps.size(), *node);
    if (!deps.empty() && (ee = cudaGraphAddDependencies_v2(gr, deps.data(), to.data(), ed.data(), deps.size())) != cudaSuccess)
      return cuda_fail(ee, "cudaGraphAddDependencies_v2");
    return KTILER_OK;
  };
  // CTA-dispatch priority per kernel node (KTILER_DAG_PRIO experiment; needs
  // cudaGraphInstantiateFlagUseNodePriority at instantiation, dag_uses_priority): 1 = the
  // deeper the node, the higher its priority, so a consumer sub-kernel's CTAs are dispatched
  // before the next fragment's source CTAs that keep refilling the SMs; 2 = the reverse.
  const int prio_mode = dag_prio_mode();
  std::vector<int> ndepth(g.nodes.size(), 0);
  for (int v : g.topo)
    for (auto& c : g.in_ch[v]) ndepth[v] = std::max(ndepth[v], ndepth[c.u] + 1);
  int prio_lo = 0, prio_hi = 0;  // least / greatest (numerically lower = higher priority)
  if (prio_mode) cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
  auto set_prio = [&](cudaGraphNode_t nd, int node) -> ktiler_status {
    if (!prio_mode || node < 0) return KTILER_OK;
    int d = ndepth[node], dmax = 0;
    for (int x : ndepth) dmax = std::max(dmax, x);
    if (prio_mode == 2) d = dmax - d;
    if (prio_mode == 3) d = d > 0 ? dmax : 0;   // source nodes low, every consumer high
    if (prio_mode == 4) d = d >= 3 ? dmax : 0;  // only the deep (quarter-resolution) consumers high
    cudaKernelNodeAttrValue v = {};
    v.priority = std::max(prio_hi, prio_lo - d);
    cudaError_t ee = cudaGraphKernelNodeSetAttribute(nd, cudaLaunchAttributePriority, &v);
    return ee == cudaSuccess ? KTILER_OK : cuda_fail(ee, "cudaGraphKernelNodeSetAttribute(priority)");
  };
  size_t li = 0;
  std::vector<std::vector<size_t>> launch_of(nsub);  // P->launches index of each node in nodes_of
  // dispatch-order edges (dag_order_edges): sub-kernel index of (fragment, node)
  const bool order = dag_order_edges(P);
  std::vector<std::vector<int>> sub_at;
  if (order) {
    sub_at.assign(S.nfrag, std::vector<int>(g.nodes.size(), -1));
    for (int i = 0; i < nsub; ++i) sub_at[S.subs[i].frag][S.subs[i].node] = i;
  }
  for (int i = 0; i < nsub; ++i) {
    std::vector<std::pair<cudaGraphNode_t, uint8_t>> dp;
    const int v = S.subs[i].node, f = S.subs[i].frag;
    if (order && g.in_ch[v].empty() && f > 0 && g.nodes[v].op != KTILER_OP_CUSTOM && g.nodes[v].wacc >= 0 &&
        !g.bufs[g.nodes[v].acc[g.nodes[v].wacc].buf].d.ring_frames) {
      std::vector<int> from;
      if (dag_order_node() >= 0 && dag_order_node() < (int)g.nodes.size()) from.push_back(dag_order_node());
      else
        for (const kt::Chan& ch : g.out_ch[v]) from.push_back(ch.v);
      for (int u : from) {
        if (g.nodes[u].op == KTILER_OP_CUSTOM) continue;  // a programmatic port needs a kernel node
        const int d = sub_at[f - 1][u];
        if (d >= 0 && d < i)
          for (size_t k = 0; k < nodes_of[d].size(); ++k) dp.push_back({nodes_of[d][k], (uint8_t)1});
      }
    }
    for (int d : edges[i]) {
      const bool prod = pdl_all || std::find(S.sub_deps[i].begin(), S.sub_deps[i].end(), d) != S.sub_deps[i].end() ||
                        (pdl_chain && S.subs[d].node == S.subs[i].node) ||
                        (pdl_window && S.subs[d].node != S.subs[i].node);
      for (size_t k = 0; k < nodes_of[d].size(); ++k)
        dp.push_back({nodes_of[d][k], (uint8_t)(pdl && prod && pdl_edge(P, P->launches[launch_of[d][k]]))});
    }
    std::sort(dp.begin(), dp.end());
    std::vector<cudaGraphNode_t> deps;
    std::vector<uint8_t> prog;
    for (size_t j = 0; j < dp.size(); ++j) {
      if (!deps.empty() && deps.back() == dp[j].first) {
        prog.back() &= dp[j].second;  // a node reached both ways: full completion wins
        continue;
      }
      deps.push_back(dp[j].first);
      prog.push_back(dp[j].second);
    }
    for (; li < P->launches.size() && P->launches[li].sub == i; ++li) {
      cudaGraphNode_t nd;
      ktiler_status st = add_node(P->launches[li], deps, prog, &nd);
      if (!st && P->launches[li].node >= 0 && P->launches[li].n->op != KTILER_OP_CUSTOM) st = set_prio(nd, P->launches[li].node);
      if (st) {
        cudaGraphDestroy(gr);
        return st;
      }
      nodes_of[i].push_back(nd);
      launch_of[i].push_back(li);
    }
  }
  for (Launch& D : P->dag_disc) {
    std::vector<cudaGraphNode_t> deps;
    for (int r : S.discard_readers[D.sub]) deps.insert(deps.end(), nodes_of[r].begin(), nodes_of[r].end());
    std::sort(deps.begin(), deps.end());
    deps.erase(std::unique(deps.begin(), deps.end()), deps.end());
    cudaGraphNode_t nd;
    ktiler_status st = add_node(D, deps, {}, &nd);
    if (st) {
      cudaGraphDestroy(gr);
      return st;
    }
  }
  *out = gr;
  return KTILER_OK;
}

ktiler_status enqueue(ktiler_plan_s* P, cudaStream_t st) {
  const Launch* prev = nullptr;  // the previous launch in the stream
  for (auto& L : P->launches) {
    if (L.node >= 0 && L.n->op == KTILER_OP_CUSTOM) {
      L.n->launch(L.n->user, L.crects.data(), (int32_t)(L.crects.size() / 6), (void*)st);
      prev = &L;
      continue;
    }
    kfn_t fn = launch_fn(L);
    int64_t grid = 0;
    ktiler_status ps = prep_launch(P, L, fn, &grid);
    if (ps) return ps;
    L.grid = grid;
    const bool prog = L.kp.pdl && prev && pdl_edge(P, *prev);
    prev = &L;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = L.block;
    cfg.dynamicSmemBytes = (size_t)L.smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[2];
    int na = 0;
    if (prog || L.kp.chain == 1) {
      attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      attr[na].val.programmaticStreamSerializationAllowed = 1;
      ++na;
    }
    if (P->pol.exec_mode == KTILER_EXEC_GRAPH_PERSIST_L2 && L.node >= 0) {
      // the sub-kernel's output region persists in L2 for its consumer; input streams
      const DBuf& o = L.kp.out;
      const LRect& r0 = L.kp.r[0];
      const LRect& r1 = L.kp.r[L.kp.nrect - 1];
      int64_t eb = L.n->op == 3 ? 4 : 1;
      uint64_t lo = (uint64_t)(o.p + r0.z0 * o.fstride + (int64_t)r0.y0 * L.kp.th * o.pitch);
      uint64_t hi = (uint64_t)(o.p + (r1.z1 - 1) * o.fstride + std::min<int64_t>((int64_t)r1.y1 * L.kp.th, o.H) * o.pitch);
      (void)eb;
      attr[na].id = cudaLaunchAttributeAccessPolicyWindow;
      attr[na].val.accessPolicyWindow.base_ptr = (void*)lo;
      attr[na].val.accessPolicyWindow.num_bytes = (size_t)std::min<uint64_t>(hi - lo, 64ull << 20);
      attr[na].val.accessPolicyWindow.hitRatio = 1.0f;
      attr[na].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      attr[na].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
      ++na;
    }
    cfg.attrs = na ? attr : nullptr;
    cfg.numAttrs = na;
    cudaError_t e = cudaLaunchKernelEx(&cfg, fn, L.kp);
    if (e != cudaSuccess) return cuda_fail(e, "sub-kernel launch");
  }
  if (P->pol.exec_mode == KTILER_EXEC_GRAPH_CHAIN) {
    for (auto& T : P->chain_tail) {
      const int64_t lines = T.kp.ndisc ? T.kp.dpre[T.kp.ndisc] : 0;
      const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(1184, (lines + 255) / 256));
      chain_tail_kernel<<<grid, 256, 0, st>>>(T.kp);
    }
    chain_epoch_kernel<<<1, 1, 0, st>>>(P->epoch);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "chain tail launch");
  }
  return KTILER_OK;
}

// GRAPH_CHAIN setup (first execute): device flags/counters, per-launch producer maps, and
// placement of each discard list on a later launch that first waits for the prefix flag of
// the list's last reader launch (lines are only dropped once nobody can still read them).
ktiler_status setup_chain(ktiler_plan_s* P) {
  const kt::Graph& g = P->g;
  const int nn = (int)g.nodes.size();
  if (P->has_custom) return fail(KTILER_E_UNSUPPORTED, "GRAPH_CHAIN runs built-in ops only");
  std::vector<int64_t> flag0(nn);
  int64_t nflags = 0;
  for (int v = 0; v < nn; ++v) {
    flag0[v] = nflags;
    nflags += g.nodes[v].nblocks;
  }
  const int64_t nl = (int64_t)P->launches.size();
  const size_t bytes = (size_t)(1 + nflags + 2 * nl + 64) * 4;
  char* d = nullptr;
  cudaError_t e = cudaMalloc(&d, bytes);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (chain flags)");
  P->cmem = d;
  if ((e = cudaMemset(d, 0, bytes)) != cudaSuccess) return cuda_fail(e, "cudaMemset");
  unsigned int* u = (unsigned int*)d;
  const unsigned int one = 1;
  if ((e = cudaMemcpy(u, &one, 4, cudaMemcpyHostToDevice)) != cudaSuccess) return cuda_fail(e, "cudaMemcpy");
  P->epoch = u;
  unsigned int* flags = u + 1;
  unsigned int* dcount = flags + nflags;
  unsigned int* prefix = dcount + nl;
  std::vector<int64_t> last_launch_of_sub(P->s.subs.size(), -1);
  for (int64_t l = 0; l < nl; ++l) {
    Launch& L = P->launches[l];
    const kt::Node& n = g.nodes[L.node];
    const kt::Access& r = n.acc[n.racc];
    KParams& k = L.kp;
    k.chain = l == 0 ? 2 : 1;
    k.pdl = 0;
    k.gx = (int32_t)n.gx();
    k.gy = (int32_t)n.gy();
    k.flags = flags + flag0[L.node];
    k.epoch = P->epoch;
    k.dcount = dcount + l;
    k.prefix = prefix + l;
    k.pgx = 0;
    for (auto& c : g.in_ch[L.node]) {
      const kt::Node& pu = g.nodes[c.u];
      const kt::Access& uw = pu.acc[c.w];
      k.pgx = (int32_t)pu.gx();
      k.pgy = (int32_t)pu.gy();
      k.pflags = flags + flag0[c.u];
      k.rax = (int32_t)r.ax; k.ray = (int32_t)r.ay; k.rox = (int32_t)r.ox; k.roy = (int32_t)r.oy;
      k.rhl = r.hl; k.rhr = r.hr; k.rht = r.ht; k.rhb = r.hb;
      k.wax = (int32_t)uw.ax; k.way = (int32_t)uw.ay;
    }
    last_launch_of_sub[L.sub] = l;
  }
  // discard lists: list D (dead after sub-kernel D.sub) goes to the first launch of a
  // sub-kernel >= D.sub + 2 without discards of its own, else to the tail
  int64_t next = 0;
  for (auto& D : P->dag_disc) {
    const int64_t wait_l = last_launch_of_sub[D.sub];
    while (next < nl && (P->launches[next].sub < D.sub + 2 || P->launches[next].kp.ndisc)) ++next;
    KParams* k = nullptr;
    if (next < nl) {
      k = &P->launches[next].kp;
    } else {
      Launch T;
      std::memset(&T.kp, 0, sizeof(T.kp));
      P->chain_tail.push_back(T);
      k = &P->chain_tail.back().kp;
    }
    k->ndisc = D.kp.ndisc;
    std::memcpy(k->d, D.kp.d, sizeof(k->d));
    std::memcpy(k->dpre, D.kp.dpre, sizeof(k->dpre));
    k->disc_prefix = prefix + wait_l;
  }
  if (P->chain_tail.empty()) {
    Launch T;
    std::memset(&T.kp, 0, sizeof(T.kp));
    P->chain_tail.push_back(T);
  }
  for (auto& T : P->chain_tail) {
    T.kp.epoch = P->epoch;
    T.kp.disc_prefix = prefix + (nl - 1);  // the tail waits for the whole chain
  }
  P->dag_disc.clear();
  return KTILER_OK;
}

// KTILER_PF_HALO_DISCARD (A44): blur5 / sobel3 launches of a tiled plan
// whose input is an internal buffer they alone read get a reader count per producer block
// (consumer blocks whose declared read rect meets it: Graph::consumers) and zeroed counters.
ktiler_status setup_halo_discard(ktiler_plan_s* P) {
  const kt::Graph& g = P->g;
  if (!(P->pol.flags & KTILER_PF_HALO_DISCARD) || P->s.nfrag <= 1) return KTILER_OK;
  std::vector<std::pair<unsigned int*, const uint8_t*>> per_node(g.nodes.size(), {nullptr, nullptr});
  for (auto& L : P->launches) {
    if (L.node < 0 || L.n->scalar || (L.n->op != KTILER_OP_BLUR5 && L.n->op != KTILER_OP_SOBEL3)) continue;
    const kt::Node& n = g.nodes[L.node];
    const kt::Access& r = n.acc[n.racc];
    const kt::Buffer& ib = g.bufs[r.buf];
    if (!(ib.d.flags & KTILER_BUF_INTERNAL) || ib.readers.size() != 1 || !discardable(ib) || ib.writer < 0) continue;
    const kt::Chan* ch = nullptr;
    for (const kt::Chan& c : g.in_ch[L.node])
      if (c.buf == r.buf) ch = &c;
    if (!ch) continue;
    const kt::Node& u = g.nodes[ch->u];
    const kt::Access& uw = u.acc[ch->w];
    if (g.nodes[ch->u].op == KTILER_OP_CUSTOM || u.gx() > (1 << 20) || u.gy() > (1 << 20)) continue;
    auto& slot = per_node[L.node];
    if (!slot.first) {
      const int64_t gx = u.gx(), gy = u.gy(), gz = u.gz();
      std::vector<uint8_t> need((size_t)(gx * gy));
      for (int64_t py = 0; py < gy; ++py)
        for (int64_t px = 0; px < gx; ++px) {
          const kt::BRange c = g.consumers(*ch, px, py);
          const int64_t k = c.empty() ? 0 : (c.x1 - c.x0) * (c.y1 - c.y0);
          if (k > 255) return fail(KTILER_E_UNSUPPORTED, "consumer discard: more than 255 readers of one block");
          need[(size_t)(py * gx + px)] = (uint8_t)k;
        }
      void* cnt = nullptr;
      void* nd = nullptr;
      cudaError_t e = cudaMalloc(&cnt, (size_t)(gx * gy * gz) * 4);
      if (e == cudaSuccess) e = cudaMalloc(&nd, need.size());
      if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (halo-reader counters)");
      P->hmem.push_back(cnt);
      P->hmem.push_back(nd);
      if ((e = cudaMemset(cnt, 0, (size_t)(gx * gy * gz) * 4)) != cudaSuccess) return cuda_fail(e, "cudaMemset");
      if ((e = cudaMemcpy(nd, need.data(), need.size(), cudaMemcpyHostToDevice)) != cudaSuccess)
        return cuda_fail(e, "cudaMemcpy");
      slot = {(unsigned int*)cnt, (const uint8_t*)nd};
    }
    KParams& k = L.kp;
    k.hcnt = slot.first;
    k.hneed = slot.second;
    k.pgx = (int32_t)u.gx();
    k.pgy = (int32_t)u.gy();
    k.rax = (int32_t)r.ax; k.ray = (int32_t)r.ay; k.rox = (int32_t)r.ox; k.roy = (int32_t)r.oy;
    k.rhl = r.hl; k.rhr = r.hr; k.rht = r.ht; k.rhb = r.hb;
    k.wax = (int32_t)uw.ax; k.way = (int32_t)uw.ay;
  }
  return KTILER_OK;
}

ktiler_status setup_persistent(ktiler_plan_s* P) {
  const kt::Graph& g = P->g;
  const kt::Schedule& S = P->s;
  const int nn = (int)g.nodes.size();
  const int nsub = (int)S.subs.size();
  for (auto& n : g.nodes)
    if (n.op == KTILER_OP_CUSTOM || n.op == KTILER_OP_JACOBI || n.op == KTILER_OP_GAUSS_F32)
      return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode runs the image-pipeline built-ins (GRAY..THRESH) only");
  if (nn > PMAX_NODES) return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode: at most 8 nodes");
  std::vector<PNode> pn(nn);
  for (int v = 0; v < nn; ++v) {
    const kt::Node& n = g.nodes[v];
    const kt::Access& w = n.acc[n.wacc];
    const kt::Access& r = n.acc[n.racc];
    if (n.gx() >= (1 << 14) || n.gy() >= (1 << 14) || n.gz() > 4096)
      return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode: grid exceeds the ticket (2^14 blocks per axis, 4096 frames)");
    PNode& q = pn[v];
    std::memset(&q, 0, sizeof(q));
    q.in = dbuf(g.bufs[r.buf]);
    q.out = dbuf(g.bufs[w.buf]);
    q.op = n.op;
    q.scalar = n.scalar;
    q.tw = (int32_t)w.ax;
    q.th = (int32_t)w.ay;
    q.T = n.T;
    q.use_tmap = !n.scalar && make_tmap(g, n, &q.tmap, &q.box_bytes);
    if (!n.scalar && !q.use_tmap) return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode: input tile map unavailable");
    static const int evict_env = getenv("KTILER_EVICT_READS") ? atoi(getenv("KTILER_EVICT_READS")) : -1;
    q.in_stream = (evict_env >= 0 ? evict_env != 0 : (S.nfrag > 1 && g.bufs[r.buf].readers.size() == 1)) ||
                  !g.written_by_node(r.buf);  // as for launches
  }
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, P->device);
  int slot = 0;
  for (auto& n : g.nodes) {
    const kt::Access& w = n.acc[n.wacc];
    if (!n.scalar) slot = std::max(slot, (ktd::stage_bytes(n.op, (int)w.ax, (int)w.ay) + 127) & ~127);
  }
  int smem_sm = 0, smem_blk = 0;
  cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, P->device);
  cudaDeviceGetAttribute(&smem_blk, cudaDevAttrMaxSharedMemoryPerBlockOptin, P->device);
  cudaFuncAttributes fa{};
  auto per_cta_of = [&](void (*f)(PParams), int minb) {
    cudaFuncGetAttributes(&fa, (const void*)f);
    return std::min(smem_sm / minb - 1024, smem_blk) - (int)fa.sharedSizeBytes;
  };
  {
    // KTILER_PERSIST_GROUPS: compute groups per CTA (4 -> one CTA per SM; 2 -> two; 1 ->
    // three single-group CTAs)
    const char* ev = getenv("KTILER_PERSIST_GROUPS");
    const int ng = ev ? atoi(ev) : PERSIST_GROUPS_DEFAULT;
    if (ng >= 4) { P->pfn = persistent_kernel<4, 1>; P->pminb = 1; P->pgroups = 4; }
    else if (ng == 2) { P->pfn = persistent_kernel<2, 2>; P->pminb = 2; P->pgroups = 2; }
    else { P->pfn = persistent_kernel<1, 3>; P->pminb = 3; P->pgroups = 1; }
    // tiles too large for two slots per compute group (e.g. 64 KB f32 thresh tiles): one
    // single-group CTA per SM (the whole shared memory for its ring)
    if (!ev && slot && per_cta_of(P->pfn, P->pminb) / slot < 2 * P->pgroups) {
      P->pfn = persistent_kernel<1, 1>;
      P->pminb = 1;
      P->pgroups = 1;
    }
    P->pthreads = P->pgroups * PCOMP_THREADS + 64;
  }
  // ring depth: as many slots as fit the shared memory of MINB CTAs per SM, a multiple of
  // the compute groups (slot s always serves group s mod NG, so every waiter on a slot's
  // barrier has consumed the slot's previous use itself: no parity aliasing)
  const int per_cta = per_cta_of(P->pfn, P->pminb);
  const int ngr = P->pgroups;
  int nslots = slot ? std::min(PSTAGES_MAX, std::max(2 * ngr, per_cta / slot)) : 2 * ngr;
  if (const char* ev = getenv("KTILER_PERSIST_SLOTS")) nslots = std::min(PSTAGES_MAX, std::max(ngr, atoi(ev)));
  nslots -= nslots % ngr;
  P->psmem = std::max(slot, 128) * nslots;
  if (P->psmem + (int)fa.sharedSizeBytes > smem_blk)
    return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode: staging slots exceed shared memory");
  if (P->psmem + (int)fa.sharedSizeBytes > 48 * 1024) {
    cudaError_t ea = cudaFuncSetAttribute((const void*)P->pfn, cudaFuncAttributeMaxDynamicSharedMemorySize, P->psmem);
    if (ea != cudaSuccess) return cuda_fail(ea, "cudaFuncSetAttribute (persistent smem)");
  }
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, P->pfn, P->pthreads, P->psmem);
  if (occ < 1) return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode: kernel does not fit an SM");
  P->pctas = P->pol.persistent_ctas > 0 ? std::min(P->pol.persistent_ctas, nsm * occ) : nsm * occ;
  // Ticket order, in pipeline steps.  skew < 0: the emitted (fragment-major) order, one
  // sub-kernel per step.  skew = k > 0: software pipeline over fragments — the
  // sub-kernel of fragment f at node depth d runs in step f + d*k.  A consumer's
  // producers sit in fragments <= f at smaller depth, hence in steps at least k earlier:
  // still a valid total order, and the sub-kernels of one step never
  // depend on each other, so their tiles are interleaved evenly (memory-bound and
  // ALU-bound tiles of different fragments share every SM) and a step only waits for
  // the step k before it.
  std::vector<int> depth(nn, 0);
  int dmax = 0;
  for (int v : g.topo)
    for (auto& c : g.in_ch[v]) depth[v] = std::max(depth[v], depth[c.u] + 1);
  for (int v = 0; v < nn; ++v) dmax = std::max(dmax, depth[v]);
  const int64_t nfrag = S.nfrag;
  std::vector<std::vector<int>> by_frag(nfrag, std::vector<int>(nn, -1));
  for (int i = 0; i < nsub; ++i) by_frag[S.subs[i].frag][S.subs[i].node] = i;
  int64_t k = P->pol.pipeline_skew;
  if (k == 0) k = 1;
  P->skew = k;
  const char* ie = getenv("KTILER_PERSIST_INTERLEAVE");
  const bool interleave = k > 0 && ie && atoi(ie) != 0;  // opt-in: mixed ops thrash the instruction cache
  std::vector<std::vector<int>> steps;  // sub-kernels per step
  std::vector<int> step_of(nsub, 0);
  if (k < 0) {
    for (int i = 0; i < nsub; ++i) steps.push_back({i});
  } else {
    std::vector<int> rtopo(g.topo.rbegin(), g.topo.rend());
    for (int64_t st = 0; st < nfrag + dmax * k; ++st) {
      steps.emplace_back();
      for (int v : rtopo) {
        const int64_t f = st - depth[v] * k;
        if (f >= 0 && f < nfrag && by_frag[f][v] >= 0) steps.back().push_back(by_frag[f][v]);
      }
    }
  }
  for (size_t st = 0; st < steps.size(); ++st)
    for (int i : steps[st]) step_of[i] = (int)st;
  // Discard lists (groups nsub + si): at the end of the step of their last reader, after
  // the step's source tiles (deepest node first: the readers come early in the step), or
  // nn sub-kernels later in fragment-major order.  Measured on B200: the L2 writes dirty
  // lines back on its own within microseconds, so a discard a whole step late saves
  // nothing — dead lines must go as soon as their readers are done.
  const bool disc = (P->pol.flags & KTILER_PF_DISCARD_DEAD) != 0;
  const char* dl = getenv("KTILER_PERSIST_DLAG");
  const int dlag = k < 0 ? nn : (dl ? atoi(dl) : 0);
  std::vector<std::vector<int>> disc_in(steps.size() + dlag + 1);
  std::vector<DRect> drects;
  std::vector<std::vector<int>> drect_of(nsub);
  if (disc) {
    for (int si = 0; si < nsub; ++si) {
      for (auto& dd : S.discards[si]) {
        if (!discardable(g.bufs[dd.buf])) continue;
        DRect dr = drect(g, dd);
        if (dr.lpr <= 0) continue;
        drect_of[si].push_back((int)drects.size());
        drects.push_back(dr);
      }
      if (drect_of[si].empty()) continue;
      int last = step_of[si];
      for (int r : S.discard_readers[si]) last = std::max(last, step_of[r]);
      disc_in[std::min<size_t>(disc_in.size() - 1, (size_t)last + dlag)].push_back(si);
    }
  }
  // groups' dependency lists (CSR)
  const int ngroups = 2 * nsub;
  if (ngroups >= (1 << PGROUP_BITS)) return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode: too many sub-kernels");
  std::vector<int32_t> dep_off(ngroups + 1, 0);
  std::vector<PDep> deps;
  for (int gi = 0; gi < ngroups; ++gi) {
    const std::vector<int32_t>& src = gi < nsub ? S.sub_deps[gi] : S.discard_readers[gi - nsub];
    for (int32_t u : src) deps.push_back(PDep{u, (uint32_t)S.subs[u].nblocks});
    dep_off[gi + 1] = (int32_t)deps.size();
  }
  // the tickets in global order: per step, each member's tickets spread evenly over the
  // step (key (j + 1/2) / n), discard chunks likewise
  std::vector<uint64_t> tickets;
  std::vector<PChunk> chunks;
  constexpr int64_t CHUNK_LINES = 2048;  // 256 KB of dead lines per discard ticket
  std::vector<std::pair<double, uint64_t>> keyed;
  auto put = [&](std::vector<uint64_t>& v) {
    const double n = (double)v.size();
    for (size_t j = 0; j < v.size(); ++j) keyed.push_back({interleave ? (j + 0.5) / n : 0.0, v[j]});
  };
  std::vector<uint64_t> tmp;
  for (size_t st = 0; st < disc_in.size(); ++st) {
    keyed.clear();
    if (st < steps.size())
      for (int si : steps[st]) {
        tmp.clear();
        const kt::SubKernel& sk = S.subs[si];
        for (auto& r : sk.rects)
          for (int64_t z = r.z0; z < r.z1; ++z)
            for (int64_t y = r.y0; y < r.y1; ++y)
              for (int64_t x = r.x0; x < r.x1; ++x)
                tmp.push_back(pack_ticket((uint64_t)sk.node, (uint64_t)si, tile_payload(x, y, z)));
        put(tmp);
      }
    // the step's discard chunks after its tiles (non-interleaved): the lines die as soon
    // as possible while the readers (a step earlier) have had a whole step to finish
    for (int si : disc_in[st]) {
      tmp.clear();
      for (int di : drect_of[si]) {
        const DRect& r = drects[di];
        const int64_t lines = r.lpr * (int64_t)(r.y1 - r.y0) * (r.z1 - r.z0);
        for (int64_t l0 = 0; l0 < lines; l0 += CHUNK_LINES) {
          tmp.push_back(pack_ticket(PK_DISCARD, (uint64_t)(nsub + si), chunks.size()));
          chunks.push_back(PChunk{di, (int32_t)std::min(CHUNK_LINES, lines - l0), l0});
        }
      }
      put(tmp);
    }
    std::stable_sort(keyed.begin(), keyed.end(),
                     [](const std::pair<double, uint64_t>& a, const std::pair<double, uint64_t>& b) { return a.first < b.first; });
    for (auto& kv : keyed) tickets.push_back(kv.second);
  }
  // Static: per-CTA contiguous ticket lists (ticket i -> CTA i mod G, in order),
  // STOP-padded; the first ticket of each group in a CTA's list carries PK_CHECK.
  // Dynamic (default; KTILER_PERSIST_DYNAMIC=0 for static): the global order as is; CTAs claim chunks of it
  // from an atomic counter (load balance), checking dependencies through a group cache.
  const int64_t G = P->pctas, T = (int64_t)tickets.size();
  const char* dy = getenv("KTILER_PERSIST_DYNAMIC");
  const bool dynamic = !dy || atoi(dy) != 0;  // default on: load-balanced claims
  if (T >= (1ll << 31)) return fail(KTILER_E_UNSUPPORTED, "PERSISTENT mode: more than 2^31 tickets");
  const int64_t per = dynamic ? 0 : (T + G - 1) / G + 1;
  std::vector<uint64_t> desc;
  if (dynamic) {
    desc = tickets;
  } else {
    desc.assign((size_t)(G * per), pack_ticket(PK_STOP, 0, 0));
    for (int64_t i = 0; i < T; ++i) desc[(size_t)((i % G) * per + i / G)] = tickets[(size_t)i];
    std::vector<int64_t> stamp(ngroups, -1);
    for (int64_t c = 0; c < G; ++c)
      for (int64_t j = 0; j < per; ++j) {
        uint64_t& d = desc[(size_t)(c * per + j)];
        if ((d >> 60) == PK_STOP) break;
        const int gr = ticket_group(d);
        if (stamp[gr] != c && dep_off[gr + 1] > dep_off[gr]) d |= PK_CHECK;
        stamp[gr] = c;
      }
  }
  // one device allocation: ctrl | counters | dep_off | deps | drects | chunks | nodes | desc
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  size_t o_ctrl = 0, o_cnt = al(sizeof(PCtrl)), o_doff = o_cnt + al((size_t)nsub * 4 + 4);
  size_t o_deps = o_doff + al(dep_off.size() * 4), o_dr = o_deps + al(deps.size() * sizeof(PDep) + 8);
  size_t o_ch = o_dr + al(drects.size() * sizeof(DRect) + 8), o_nodes = o_ch + al(chunks.size() * sizeof(PChunk) + 8);
  size_t o_desc = o_nodes + al(pn.size() * sizeof(PNode)), total = o_desc + al(desc.size() * sizeof(uint64_t));
  char* d = nullptr;
  cudaError_t e = cudaMalloc(&d, total);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (persistent tables)");
  P->dmem = d;
  PCtrl c0{0, 1, 0, 0};  // done, epoch, ticket
  if ((e = cudaMemset(d, 0, total)) != cudaSuccess) return cuda_fail(e, "cudaMemset");
  cudaMemcpy(d + o_ctrl, &c0, sizeof(c0), cudaMemcpyHostToDevice);
  cudaMemcpy(d + o_doff, dep_off.data(), dep_off.size() * 4, cudaMemcpyHostToDevice);
  if (!deps.empty()) cudaMemcpy(d + o_deps, deps.data(), deps.size() * sizeof(PDep), cudaMemcpyHostToDevice);
  if (!drects.empty()) cudaMemcpy(d + o_dr, drects.data(), drects.size() * sizeof(DRect), cudaMemcpyHostToDevice);
  if (!chunks.empty()) cudaMemcpy(d + o_ch, chunks.data(), chunks.size() * sizeof(PChunk), cudaMemcpyHostToDevice);
  cudaMemcpy(d + o_nodes, pn.data(), pn.size() * sizeof(PNode), cudaMemcpyHostToDevice);
  if ((e = cudaMemcpy(d + o_desc, desc.data(), desc.size() * sizeof(uint64_t), cudaMemcpyHostToDevice)) != cudaSuccess)
    return cuda_fail(e, "cudaMemcpy (persistent tables)");
  P->pp.nodes = (const PNode*)(d + o_nodes);
  P->pp.desc = (const uint64_t*)(d + o_desc);
  P->pp.per_cta = per;
  P->pp.total = T;
  P->pp.dep_off = (const int32_t*)(d + o_doff);
  P->pp.deps = (const PDep*)(d + o_deps);
  P->pp.drects = (const DRect*)(d + o_dr);
  P->pp.chunks = (const PChunk*)(d + o_ch);
  P->pp.nsub = nsub;
  P->pp.cnt = (unsigned int*)(d + o_cnt);
  P->pp.ctrl = (PCtrl*)(d + o_ctrl);
  P->pp.stage_bytes = std::max(slot, 128);
  P->pp.nslots = nslots;
  P->pp.nnodes = nn;
  return KTILER_OK;
}


// ------------------------------------------------------------------------------------
// KTILER_EXEC_FLOW setup (flow.cuh): node table, global pipelined order, role ticket
// lists, run-ahead window, slot -> role map, kernel variant and ring depth.
// ------------------------------------------------------------------------------------
typedef void (*ffn_t)(ktflow::FParams);
ffn_t flow_variant(int k) {
  switch (k) {
    case 1: return ktflow::flow_kernel<8, 1>;  // tiles too large for two slots at 2 CTAs / SM
    case 2: return ktflow::flow_kernel<8, 2>;
    case 3: return ktflow::flow_kernel<4, 3>;
    case 5: return ktflow::flow_kernel<3, 5>;
    default: return ktflow::flow_kernel<4, 4>;
  }
}
int flow_threads(int k) { return k == 5 ? 128 : (k <= 2 ? 288 : 160); }

// Automatic roles: ONE role serving every node, on K slots per SM.  Measured on 16 x 8K
// (profiles/r02_flow_sweeps.txt): a CTA that can take any ready tile keeps its warps busy;
// per-node roles leave the issue-bound nodes (blur, sobel) with a few warps per SM and
// multi-node roles without the others' tiles stall on their own dependencies.
void flow_auto_roles(const kt::Graph& g, int K, std::vector<int32_t>& node_role, std::vector<int32_t>& slot_role) {
  node_role.assign(g.nodes.size(), 0);
  slot_role.assign(K, 0);
}

ktiler_status setup_flow(ktiler_plan_s* P) {
  using namespace ktflow;
  const kt::Graph& g = P->g;
  const kt::Schedule& S = P->s;
  const int nn = (int)g.nodes.size();
  const int nsub = (int)S.subs.size();
  if (nn > FMAX_NODES) return fail(KTILER_E_UNSUPPORTED, "FLOW mode: at most 1024 nodes");
  for (auto& n : g.nodes) {
    if (n.op == KTILER_OP_CUSTOM || n.scalar)
      return fail(KTILER_E_UNSUPPORTED, "FLOW mode runs the vector built-ins only (no OP_CUSTOM, no one-thread-per-pixel)");
    if (n.gx() > FLOW_BXY_MAX + 1 || n.gy() > FLOW_BXY_MAX + 1 || n.gz() > FLOW_BZ_MAX + 1)
      return fail(KTILER_E_UNSUPPORTED, "FLOW mode: grid exceeds the ticket (4096 blocks per axis, 256 frames)");
  }
  // ---- node table ----
  std::vector<int64_t> flag0(nn);
  int64_t nflags = 0;
  for (int v = 0; v < nn; ++v) {
    flag0[v] = nflags;
    nflags += g.nodes[v].nblocks;
  }
  std::vector<FNode> fnodes(nn);

  for (int v = 0; v < nn; ++v) {
    const kt::Node& n = g.nodes[v];
    const kt::Access& w = n.acc[n.wacc];
    const kt::Access& r = n.acc[n.racc];
    FNode& q = fnodes[v];
    std::memset(&q, 0, sizeof(q));
    if (!make_tmap(g, n, &q.tmap, &q.box_bytes)) return fail(KTILER_E_UNSUPPORTED, "FLOW mode: input tile map unavailable");
    q.in = dbuf(g.bufs[r.buf]);
    q.out = dbuf(g.bufs[w.buf]);
    if (n.racc2 >= 0) q.aux = dbuf(g.bufs[n.acc[n.racc2].buf]);
    q.radius = n.radius;
    for (int k = 0; k < 9; ++k) q.taps[k] = n.taps[k];
    q.flag0 = flag0[v];
    q.op = n.op;
    q.tw = (int32_t)w.ax;
    q.th = (int32_t)w.ay;
    q.T = n.T;
    q.gx = (int32_t)n.gx();
    q.gy = (int32_t)n.gy();
    q.leaf = g.out_ch[v].empty();
    const kt::Buffer& ib = g.bufs[r.buf];
    // evict-first reads: the graph input, and intermediates with one reader node (DESIGN A42)
    q.in_stream = ib.readers.size() == 1 || !g.written_by_node(r.buf);
    q.cdisc = (P->pol.flags & KTILER_PF_CONSUMER_DISCARD) && (n.op == KTILER_OP_DOWN2 || n.op == KTILER_OP_THRESH) &&
              (ib.d.flags & KTILER_BUF_INTERNAL) && ib.readers.size() == 1 && !r.hl && !r.hr && !r.ht && !r.hb &&
              discardable(ib) && g.written_by_node(r.buf);
    if (g.in_ch[v].size() > 1) return fail(KTILER_E_UNSUPPORTED, "FLOW mode: one producer per node");
    for (auto& c : g.in_ch[v]) {
      const kt::Node& pu = g.nodes[c.u];
      const kt::Access& uw = pu.acc[c.w];
      q.pflag0 = flag0[c.u];
      q.pgx = (int32_t)pu.gx();
      q.pgy = (int32_t)pu.gy();
      q.rax = (int32_t)r.ax; q.ray = (int32_t)r.ay; q.rox = (int32_t)r.ox; q.roy = (int32_t)r.oy;
      q.rhl = r.hl; q.rhr = r.hr; q.rht = r.ht; q.rhb = r.hb;
      q.wax = (int32_t)uw.ax; q.way = (int32_t)uw.ay;
    }

  }
  // ---- kernel variant, slots (CTAs) per SM, shared memory per CTA ----
  int K = (int)P->flow_slot_role.size();
  if (P->flow_slot_role.empty()) {
    // automatic: as many CTAs per SM as leave room for two staging slots of the largest
    // tile each (more compute warps per SM; 3 for the shipped geometry's 37 KB blur tiles)
    int maxst = 128;
    for (auto& n : g.nodes) {
      const kt::Access& w = n.acc[n.wacc];
      maxst = std::max(maxst, (ktd::stage_bytes(n.op, (int)w.ax, (int)w.ay) + 127) & ~127);
    }
    int smem_sm0 = 0;
    cudaDeviceGetAttribute(&smem_sm0, cudaDevAttrMaxSharedMemoryPerMultiprocessor, P->device);
    K = 1;
    for (int k = 5; k >= 2; --k)
      if (smem_sm0 / k - 1024 - 1024 >= 2 * maxst) {
        K = k;
        break;
      }
  }
  if (K < 1 || K > 5) return fail(KTILER_E_UNSUPPORTED, "FLOW mode: 1..5 slots (CTAs) per SM");
  P->ffn = flow_variant(K);
  P->fthreads = flow_threads(K);
  int nsm = 0, smem_sm = 0, smem_blk = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, P->device);
  cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, P->device);
  cudaDeviceGetAttribute(&smem_blk, cudaDevAttrMaxSharedMemoryPerBlockOptin, P->device);
  cudaFuncAttributes fa{};
  cudaFuncGetAttributes(&fa, (const void*)P->ffn);
  P->fsmem = (std::min(smem_sm / K - 1024, smem_blk) - (int)fa.sharedSizeBytes) & ~127;
  {  // static + dynamic may pass the 48 KB default
    cudaError_t ea = cudaFuncSetAttribute((const void*)P->ffn, cudaFuncAttributeMaxDynamicSharedMemorySize, P->fsmem);
    if (ea != cudaSuccess) return cuda_fail(ea, "cudaFuncSetAttribute (flow smem)");
  }
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, P->ffn, P->fthreads, P->fsmem);
  if (occ < K) return fail(KTILER_E_UNSUPPORTED, "FLOW mode: " + std::to_string(K) + " CTAs do not fit an SM (" +
                                                     std::to_string(occ) + ")");
  P->fctas = nsm * K;
  // ---- roles ----
  std::vector<int32_t> node_role = P->flow_node_role, slot_role = P->flow_slot_role;
  if (node_role.empty() || slot_role.empty()) flow_auto_roles(g, K, node_role, slot_role);
  if ((int)node_role.size() != nn) return fail(KTILER_E_INVALID, "FLOW roles: one role per node");
  int nroles = 0;
  for (int r : node_role) nroles = std::max(nroles, r + 1);
  if (nroles > FMAX_ROLES) return fail(KTILER_E_INVALID, "FLOW roles: at most 16");
  std::vector<int> served(nroles, 0);
  for (int r : slot_role) {
    if (r < 0 || r >= nroles) return fail(KTILER_E_INVALID, "FLOW roles: slot role out of range");
    served[r] = 1;
  }
  for (int r = 0; r < nroles; ++r)
    if (!served[r]) return fail(KTILER_E_INVALID, "FLOW roles: every role needs a slot");
  // ---- each role's ring: slots of its largest staged tile, as many as the CTA's smem holds ----
  std::vector<int32_t> rstage(FMAX_ROLES, 128), rslots(FMAX_ROLES, 0);
  for (int v = 0; v < nn; ++v) {
    const kt::Node& n = g.nodes[v];
    const kt::Access& w = n.acc[n.wacc];
    rstage[node_role[v]] = std::max(rstage[node_role[v]], (ktd::stage_bytes(n.op, (int)w.ax, (int)w.ay) + 127) & ~127);
  }
  int cap_slots = FSLOTS_MAX;
  if (const char* ev = getenv("KTILER_FLOW_SLOTS")) cap_slots = std::min(FSLOTS_MAX, std::max(2, atoi(ev)));
  for (int r = 0; r < nroles; ++r) {
    rslots[r] = std::min(cap_slots, P->fsmem / rstage[r]);
    if (rslots[r] < 2) return fail(KTILER_E_UNSUPPORTED, "FLOW mode: tiles too large for two staging slots per CTA");
  }
  // ---- the global order: software pipeline over fragments (A37), deepest node first ----
  std::vector<int> depth(nn, 0);
  int dmax = 0;
  for (int v : g.topo)
    for (auto& c : g.in_ch[v]) depth[v] = std::max(depth[v], depth[c.u] + 1);
  for (int v = 0; v < nn; ++v) dmax = std::max(dmax, depth[v]);
  const int64_t nfrag = S.nfrag;
  std::vector<std::vector<int>> by_frag(nfrag, std::vector<int>(nn, -1));
  for (int i = 0; i < nsub; ++i) by_frag[S.subs[i].frag][S.subs[i].node] = i;
  // skew 0 -> 32: consumers 32 fragments behind their producers in the claim order, so
  // the tiles a CTA claims are mostly ready (measured best, profiles/r02_flow_sweeps.txt)
  const int64_t k = P->pol.pipeline_skew > 0 ? P->pol.pipeline_skew : 32;
  P->skew = k;
  // run-ahead window: a source tile of fragment f waits for the leaf tiles of fragments
  // <= f - W; W > dmax * k keeps every window dependency earlier in the global order
  // window: policy.window fragments beyond the pipeline depth, or (0) as many fragments as
  // the L2 budget holds of the intermediates they write (CheckCacheConst)
  int64_t wextra = P->pol.window;
  if (wextra <= 0) {
    double inter = 0;
    for (int v = 0; v < nn; ++v)
      if (!fnodes[v].leaf) {
        const kt::Node& n = g.nodes[v];
        const kt::Access& w = n.acc[n.wacc];
        inter += (double)n.nblocks * (double)w.ax * (double)w.ay * g.bufs[w.buf].d.elem_bytes;
      }
    const double per_frag = inter / std::max<int64_t>(1, nfrag);
    wextra = per_frag > 0 ? (int64_t)std::floor((double)S.budget / per_frag) : 2;
    wextra = std::max<int64_t>(2, std::min<int64_t>(wextra, nfrag));
  }
  const int64_t W = dmax * k + wextra;
  std::vector<int64_t> leaf_upto(nfrag + 1, 0);  // leaf tiles of fragments < f
  for (int64_t f = 0; f < nfrag; ++f) {
    int64_t c = 0;
    for (int v = 0; v < nn; ++v)
      if (fnodes[v].leaf && by_frag[f][v] >= 0) c += S.subs[by_frag[f][v]].nblocks;
    leaf_upto[f + 1] = leaf_upto[f] + c;
  }
  if (leaf_upto[nfrag] > (int64_t)FLOW_WAIT_MAX) return fail(KTILER_E_UNSUPPORTED, "FLOW mode: too many leaf tiles");
  std::vector<std::vector<uint64_t>> lists(nroles);
  std::vector<int> rtopo(g.topo.rbegin(), g.topo.rend());
  for (int64_t st = 0; st < nfrag + dmax * k; ++st)
    for (int v : rtopo) {
      const int64_t f = st - depth[v] * k;
      if (f < 0 || f >= nfrag || by_frag[f][v] < 0) continue;
      const kt::SubKernel& sk = S.subs[by_frag[f][v]];
      const uint64_t wait = (depth[v] == 0 && f - W >= 0 && nn > 1) ? (uint64_t)leaf_upto[f - W + 1] : 0;
      std::vector<uint64_t>& L = lists[node_role[v]];
      for (auto& r : sk.rects)
        for (int64_t z = r.z0; z < r.z1; ++z)
          for (int64_t y = r.y0; y < r.y1; ++y)
            for (int64_t x = r.x0; x < r.x1; ++x) L.push_back(flow_ticket((uint64_t)v, wait, x, y, z));
    }
  std::vector<int64_t> role_off(nroles + 1, 0);
  for (int r = 0; r < nroles; ++r) role_off[r + 1] = role_off[r] + (int64_t)lists[r].size();
  // ---- one device allocation: ctrl | claims | smslot | slot_role | role_off | flags | nodes | tickets ----
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  const size_t o_ctrl = 0, o_claim = al(sizeof(FCtrl)), o_sms = o_claim + al(FMAX_ROLES * 4);
  const size_t o_sr = o_sms + al(256 * 4), o_ro = o_sr + al(FMAX_SLOTS * 4), o_fl = o_ro + al((nroles + 1) * 8);
  const size_t o_nd = o_fl + al((size_t)nflags * 4), o_tk = o_nd + al(fnodes.size() * sizeof(FNode));
  const size_t total = o_tk + al((size_t)role_off[nroles] * 8 + 8);
  char* d = nullptr;
  cudaError_t e = cudaMalloc(&d, total);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (flow tables)");
  P->fmem = d;
  if ((e = cudaMemset(d, 0, total)) != cudaSuccess) return cuda_fail(e, "cudaMemset");
  const FCtrl c0{1, 0, 0, 0};
  std::vector<int32_t> sr(FMAX_SLOTS, 0);
  for (size_t i = 0; i < slot_role.size(); ++i) sr[i] = slot_role[i];
  cudaMemcpy(d + o_ctrl, &c0, sizeof(c0), cudaMemcpyHostToDevice);
  cudaMemcpy(d + o_sr, sr.data(), sr.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(d + o_ro, role_off.data(), role_off.size() * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(d + o_nd, fnodes.data(), fnodes.size() * sizeof(FNode), cudaMemcpyHostToDevice);
  for (int r = 0; r < nroles; ++r)
    if (!lists[r].empty())
      cudaMemcpy(d + o_tk + role_off[r] * 8, lists[r].data(), lists[r].size() * 8, cudaMemcpyHostToDevice);
  if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e, "cudaMemcpy (flow tables)");
  FParams& fp = P->fp;
  fp.nodes = (const FNode*)(d + o_nd);
  fp.tickets = (const uint64_t*)(d + o_tk);
  fp.role_off = (const int64_t*)(d + o_ro);
  fp.slot_role = (const int32_t*)(d + o_sr);
  fp.claim = (unsigned int*)(d + o_claim);
  fp.smslot = (unsigned int*)(d + o_sms);
  fp.flags = (unsigned int*)(d + o_fl);
  fp.ctrl = (FCtrl*)(d + o_ctrl);
  for (int r = 0; r < FMAX_ROLES; ++r) {
    fp.role_stage[r] = rstage[r];
    fp.role_nslots[r] = rslots[r];
  }
  fp.nslots_sm = K;
  fp.batch = 1;  // measured best (profiles/r02_flow_sweeps.txt): claim one ticket at a time
  if (const char* ev = getenv("KTILER_FLOW_BATCH")) fp.batch = std::min(32, std::max(1, atoi(ev)));
  fp.pending = 2;
  if (const char* ev = getenv("KTILER_FLOW_PENDING")) fp.pending = std::min(32, std::max(1, atoi(ev)));
  fp.pending = std::max(fp.pending, fp.batch);
  fp.tb = ktflow::FTrace{P->tb.rec, P->tb.n, P->tb.cap};
  fp.nroles = nroles;
  fp.nnodes = nn;
  // watchdog: 2^24 sleeping polls (seconds) before a trap
  fp.spin_limit = 1ull << 24;
  P->flow_node_role = node_role;
  P->flow_slot_role = slot_role;
  return KTILER_OK;
}


// GRAPH_DAG / GRAPH_WAVE with an attached strip exchange: the exchange, stream-captured into
// a child graph, becomes a root every former root of the DAG depends on — one graph per
// execute, exchange then schedule.
ktiler_status prepend_halo(ktiler_plan_s* P, cudaGraph_t gr) {
  size_t nroot = 0;
  cudaError_t e = cudaGraphGetRootNodes(gr, nullptr, &nroot);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGraphGetRootNodes");
  std::vector<cudaGraphNode_t> roots(nroot);
  if (nroot && (e = cudaGraphGetRootNodes(gr, roots.data(), &nroot)) != cudaSuccess)
    return cuda_fail(e, "cudaGraphGetRootNodes");
  cudaStream_t cs;
  if ((e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking)) != cudaSuccess) return cuda_fail(e, "cudaStreamCreate");
  if ((e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal)) != cudaSuccess) {
    cudaStreamDestroy(cs);
    return cuda_fail(e, "cudaStreamBeginCapture");
  }
  ktiler_status s = kt::halo_exchange(P->halo_comm, P->halo_rank, P->halo_rows, cs);
  cudaGraph_t hx = nullptr;
  cudaError_t e2 = cudaStreamEndCapture(cs, &hx);
  cudaStreamDestroy(cs);
  if (s) {
    if (hx) cudaGraphDestroy(hx);
    return s;
  }
  if (e2 != cudaSuccess) return cuda_fail(e2, "cudaStreamEndCapture (halo)");
  cudaGraphNode_t xn;
  e = cudaGraphAddChildGraphNode(&xn, gr, nullptr, 0, hx);
  cudaGraphDestroy(hx);  // the node holds a copy
  if (e != cudaSuccess) return cuda_fail(e, "cudaGraphAddChildGraphNode (halo)");
  for (cudaGraphNode_t r : roots)
    if ((e = cudaGraphAddDependencies(gr, &xn, &r, 1)) != cudaSuccess) return cuda_fail(e, "cudaGraphAddDependencies");
  return KTILER_OK;
}

}  // namespace

extern "C" {

ktiler_status ktiler_plan(ktiler_graph_t gh, size_t cache_bytes, const ktiler_fragment_policy* pol, ktiler_plan_t* out) {
  if (!gh || !pol || !out) return fail(KTILER_E_INVALID, "NULL argument");
  *out = nullptr;
  kt::Graph* G = kt::graph_of(gh);
  ktiler_status s = G->finalize();
  if (s) return s;
  if (pol->exec_mode < KTILER_EXEC_STREAM || pol->exec_mode > KTILER_EXEC_FLOW)
    return fail(KTILER_E_INVALID, "unknown exec_mode");
  if (cache_bytes == 0) {
    int dev = 0, l2 = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    if (e != cudaSuccess || l2 <= 0) return cuda_fail(e, "cache_bytes = 0 needs a CUDA device to query the L2 size");
    cache_bytes = (size_t)l2;
  }
  auto t0 = std::chrono::steady_clock::now();
  ktiler_plan_s* P = nullptr;
  try {
    P = new ktiler_plan_s();
    P->g = *G;
    P->pol = *pol;
    s = kt::build_schedule(P->g, (int64_t)cache_bytes, *pol, P->s);
    if (s) {
      delete P;
      return s;
    }
    kt::compute_discards(P->g, P->s);
    s = ring_analysis(P);
    if (s) {
      delete P;
      return s;
    }
    build_launches(P);
    if (pol->exec_mode == KTILER_EXEC_GRAPH_DAG || pol->exec_mode == KTILER_EXEC_GRAPH_WAVE) fold_dag_discards(P);
  } catch (const std::bad_alloc&) {
    delete P;
    return fail(KTILER_E_NOMEM, "host allocation failed while planning");
  }
  P->plan_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  for (auto& n : P->g.nodes) P->has_custom |= (n.op == KTILER_OP_CUSTOM);
  *out = P;
  kt::clear_error();
  return KTILER_OK;
}

void ktiler_plan_destroy(ktiler_plan_t p) { delete p; }

ktiler_status ktiler_plan_reorder(ktiler_plan_t p, const int64_t* order, int64_t n) {
  if (!p || !order) return fail(KTILER_E_INVALID, "NULL argument");
  if (p->executed || p->device >= 0) return fail(KTILER_E_STATE, "reorder before the first execute");
  kt::Schedule& S = p->s;
  const int64_t nsub = (int64_t)S.subs.size();
  if (n != nsub) return fail(KTILER_E_INVALID, "order must list every sub-kernel once");
  std::vector<int64_t> pos(nsub, -1);
  for (int64_t k = 0; k < n; ++k) {
    if (order[k] < 0 || order[k] >= nsub || pos[order[k]] >= 0) return fail(KTILER_E_INVALID, "order is not a permutation");
    pos[order[k]] = k;
  }
  // a valid schedule: every sub-kernel after all sub-kernels it depends on
  for (int64_t i = 0; i < nsub; ++i)
    for (int32_t d : S.sub_deps[i])
      if (pos[d] >= pos[i])
        return fail(KTILER_E_INVALID, "order puts sub-kernel " + std::to_string(i) + " before sub-kernel " +
                                          std::to_string(d) + " it depends on (PAPER.md:271)");
  std::vector<kt::SubKernel> subs(nsub);
  for (int64_t k = 0; k < n; ++k) subs[k] = S.subs[order[k]];
  S.subs.swap(subs);
  // everything derived from the order: sub-kernel deps, last readers / discard lists, ring
  // WAR order, launches
  S.discards.clear();
  S.discard_lines = 0;
  kt::compute_discards(p->g, S);
  ktiler_status st = ring_analysis(p);
  if (st) return st;
  p->launches.clear();
  p->dag_disc.clear();
  build_launches(p);
  if (p->pol.exec_mode == KTILER_EXEC_GRAPH_DAG || p->pol.exec_mode == KTILER_EXEC_GRAPH_WAVE) fold_dag_discards(p);
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_plan_attach_halo(ktiler_plan_t p, ktiler_comm_t c, int32_t rank, int32_t halo_rows) {
  if (!p || !c || rank < 0 || halo_rows < 0) return fail(KTILER_E_INVALID, "bad argument");
  if (p->executed || p->device >= 0) return fail(KTILER_E_STATE, "attach the halo exchange before the first execute");
  p->halo_comm = c;
  p->halo_rank = rank;
  p->halo_rows = halo_rows;
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_plan_set_flow_roles(ktiler_plan_t p, const int32_t* node_role, int32_t n_nodes,
                                         const int32_t* slot_role, int32_t n_slots) {
  if (!p) return fail(KTILER_E_INVALID, "NULL plan");
  if (p->pol.exec_mode != KTILER_EXEC_FLOW) return fail(KTILER_E_STATE, "roles apply to KTILER_EXEC_FLOW plans");
  if (p->executed || p->device >= 0) return fail(KTILER_E_STATE, "roles must be set before the first execute");
  if (n_nodes == 0 && n_slots == 0) {
    p->flow_node_role.clear();
    p->flow_slot_role.clear();
    return KTILER_OK;
  }
  if (!node_role || !slot_role || n_nodes != (int32_t)p->g.nodes.size())
    return fail(KTILER_E_INVALID, "FLOW roles: one role per node");
  if (n_slots < 2 || n_slots > 5) return fail(KTILER_E_INVALID, "FLOW roles: 2..5 slots per SM");
  int32_t nroles = 0;
  for (int32_t i = 0; i < n_nodes; ++i) {
    if (node_role[i] < 0 || node_role[i] >= ktflow::FMAX_ROLES) return fail(KTILER_E_INVALID, "FLOW roles: role out of range");
    nroles = std::max(nroles, node_role[i] + 1);
  }
  std::vector<int> served(nroles, 0);
  for (int32_t i = 0; i < n_slots; ++i) {
    if (slot_role[i] < 0 || slot_role[i] >= nroles) return fail(KTILER_E_INVALID, "FLOW roles: slot role out of range");
    served[slot_role[i]] = 1;
  }
  for (int32_t r = 0; r < nroles; ++r)
    if (!served[r]) return fail(KTILER_E_INVALID, "FLOW roles: every role needs a slot");
  p->flow_node_role.assign(node_role, node_role + n_nodes);
  p->flow_slot_role.assign(slot_role, slot_role + n_slots);
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_plan_num_subkernels(ktiler_plan_t p, int64_t* n) {
  if (!p || !n) return fail(KTILER_E_INVALID, "NULL argument");
  *n = (int64_t)p->s.subs.size();
  return KTILER_OK;
}

ktiler_status ktiler_plan_num_fragments(ktiler_plan_t p, int64_t* n) {
  if (!p || !n) return fail(KTILER_E_INVALID, "NULL argument");
  *n = p->s.nfrag;
  return KTILER_OK;
}

ktiler_status ktiler_plan_get_subkernel(ktiler_plan_t p, int64_t i, ktiler_subkernel* out, int32_t* rects, int32_t cap) {
  if (!p || !out) return fail(KTILER_E_INVALID, "NULL argument");
  if (i < 0 || i >= (int64_t)p->s.subs.size()) return fail(KTILER_E_INVALID, "sub-kernel index out of range");
  const kt::SubKernel& sk = p->s.subs[i];
  out->node = sk.node;
  out->fragment = sk.frag;
  out->n_blocks = sk.nblocks;
  out->n_rects = (int32_t)sk.rects.size();
  out->cluster = sk.cluster;
  out->footprint_bytes = sk.footprint;
  if (rects)
    for (int32_t k = 0; k < cap && k < (int32_t)sk.rects.size(); ++k) {
      const kt::Rect6& r = sk.rects[k];
      int32_t v[6] = {r.x0, r.y0, r.z0, r.x1, r.y1, r.z1};
      std::memcpy(rects + 6 * k, v, sizeof(v));
    }
  return KTILER_OK;
}

ktiler_status ktiler_plan_get_stats(ktiler_plan_t p, ktiler_plan_stats* out) {
  if (!p || !out) return fail(KTILER_E_INVALID, "NULL argument");
  std::memset(out, 0, sizeof(*out));
  out->n_subkernels = (int64_t)p->s.subs.size();
  out->n_fragments = p->s.nfrag;
  out->n_launches = (p->pol.exec_mode == KTILER_EXEC_PERSISTENT || p->pol.exec_mode == KTILER_EXEC_FLOW)
                        ? 1
                        : (int64_t)(p->launches.size() + p->dag_disc.size()) +
                              (p->pol.exec_mode == KTILER_EXEC_GRAPH_CHAIN ? 2 : 0);
  out->n_discard_lines = (p->pol.flags & KTILER_PF_DISCARD_DEAD) ? p->s.discard_lines : 0;
  out->budget_bytes = p->s.budget;
  out->max_footprint_bytes = p->s.max_footprint;
  out->plan_ms = p->plan_ms;
  out->exec_mode = p->pol.exec_mode;
  return KTILER_OK;
}

ktiler_status ktiler_execute(ktiler_plan_t p, void* stream) {
  if (!p) return fail(KTILER_E_INVALID, "NULL plan");
  cudaStream_t st = (cudaStream_t)stream;
  cudaError_t e;
  if (p->sticky) return fail(KTILER_E_STATE, "plan setup failed at its first execute; destroy and re-plan");
  if (p->device < 0) {
    // the plan is marked ready only once every setup step succeeded; a failure is sticky
    // (a half-initialised PERSISTENT / CHAIN / halo-counter state must never launch)
    auto setup_failed = [&](ktiler_status s) {
      p->sticky = s;
      p->device = -1;
      return s;
    };
    if ((e = cudaGetDevice(&p->device)) != cudaSuccess) return setup_failed(cuda_fail(e, "cudaGetDevice"));
    if (p->pol.exec_mode == KTILER_EXEC_GRAPH_PERSIST_L2) {
      int maxp = 0;
      cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, p->device);
      if (maxp > 0) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp);
    }
    if (p->pol.exec_mode == KTILER_EXEC_PERSISTENT) {
      ktiler_status s = setup_persistent(p);
      if (s) return setup_failed(s);
      p->pp.tb = p->tb;
    } else if (p->pol.exec_mode == KTILER_EXEC_FLOW) {
      ktiler_status s = setup_flow(p);
      if (s) return setup_failed(s);
    } else {
      for (auto& L : p->launches)
        if (L.node >= 0 && L.n->op != KTILER_OP_CUSTOM && !L.n->scalar && L.kp.stage_bytes)
          L.kp.use_tmap = make_tmap(p->g, *L.n, &L.kp.tmap, &L.kp.box_bytes);
      {
        ktiler_status s = setup_halo_discard(p);
        if (s) return setup_failed(s);
      }
      if (p->pol.exec_mode == KTILER_EXEC_GRAPH_CHAIN) {
        ktiler_status s = setup_chain(p);
        if (s) return setup_failed(s);
      }
      int64_t lid = 0;
      for (auto& L : p->launches) {
        L.kp.tb = p->tb;
        L.kp.lid = lid++;
      }
      for (auto& L : p->dag_disc) {
        L.kp.tb = p->tb;
        L.kp.lid = lid++;
      }
    }
  }
  p->executed = true;
  if (p->halo_comm && (p->pol.exec_mode == KTILER_EXEC_STREAM || p->pol.exec_mode == KTILER_EXEC_PERSISTENT ||
                       p->pol.exec_mode == KTILER_EXEC_FLOW)) {
    ktiler_status hs = kt::halo_exchange(p->halo_comm, p->halo_rank, p->halo_rows, st);
    if (hs) return hs;
  }
  switch (p->pol.exec_mode) {
    case KTILER_EXEC_STREAM: {
      ktiler_status s = enqueue(p, st);
      if (s) return s;
      break;
    }
    case KTILER_EXEC_GRAPH_DAG:
    case KTILER_EXEC_GRAPH_WAVE: {
      if (!p->exec) {
        cudaGraph_t gr = nullptr;
        ktiler_status s = build_dag(p, &gr);
        if (s) return s;
        if (p->halo_comm && (s = prepend_halo(p, gr))) {
          cudaGraphDestroy(gr);
          return s;
        }
        p->graph = gr;
        const unsigned long long iflags = dag_prio_mode() ? cudaGraphInstantiateFlagUseNodePriority : 0;
        if ((e = cudaGraphInstantiate(&p->exec, gr, iflags)) != cudaSuccess) return cuda_fail(e, "cudaGraphInstantiate");
      }
      if ((e = cudaGraphLaunch(p->exec, st)) != cudaSuccess) return cuda_fail(e, "cudaGraphLaunch");
      break;
    }
    case KTILER_EXEC_GRAPH:
    case KTILER_EXEC_GRAPH_CHAIN:
    case KTILER_EXEC_GRAPH_PERSIST_L2: {
      if (!p->exec) {
        cudaStream_t cs;
        if ((e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking)) != cudaSuccess) return cuda_fail(e, "cudaStreamCreate");
        if ((e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal)) != cudaSuccess) {
          cudaStreamDestroy(cs);
          return cuda_fail(e, "cudaStreamBeginCapture");
        }
        ktiler_status s = p->halo_comm ? kt::halo_exchange(p->halo_comm, p->halo_rank, p->halo_rows, cs) : KTILER_OK;
        if (!s) s = enqueue(p, cs);
        cudaGraph_t gr = nullptr;
        cudaError_t e2 = cudaStreamEndCapture(cs, &gr);
        cudaStreamDestroy(cs);
        if (s) {
          if (gr) cudaGraphDestroy(gr);
          return s;
        }
        if (e2 != cudaSuccess) return cuda_fail(e2, "cudaStreamEndCapture");
        p->graph = gr;
        if ((e = cudaGraphInstantiate(&p->exec, gr, 0)) != cudaSuccess) return cuda_fail(e, "cudaGraphInstantiate");
      }
      if ((e = cudaGraphLaunch(p->exec, st)) != cudaSuccess) return cuda_fail(e, "cudaGraphLaunch");
      break;
    }
    case KTILER_EXEC_PERSISTENT: {
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3((unsigned)p->pctas);
      cfg.blockDim = dim3((unsigned)p->pthreads);
      cfg.dynamicSmemBytes = (size_t)p->psmem;
      cfg.stream = st;
      if ((e = cudaLaunchKernelEx(&cfg, p->pfn, p->pp)) != cudaSuccess) return cuda_fail(e, "persistent launch");
      break;
    }
    case KTILER_EXEC_FLOW: {
      // cooperative: every role's CTAs are guaranteed co-resident (flow.cuh, deadlock freedom)
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3((unsigned)p->fctas);
      cfg.blockDim = dim3((unsigned)p->fthreads);
      cfg.dynamicSmemBytes = (size_t)p->fsmem;
      cfg.stream = st;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeCooperative;
      at[0].val.cooperative = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      if ((e = cudaLaunchKernelEx(&cfg, p->ffn, p->fp)) != cudaSuccess) return cuda_fail(e, "flow launch");
      break;
    }
  }
  if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e, "launch");
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_execute_host(ktiler_plan_t p, const ktiler_host_copy* in, int32_t nin, const ktiler_host_copy* outc,
                                  int32_t nout, void* stream) {
  if (!p) return fail(KTILER_E_INVALID, "NULL plan");
  cudaStream_t st = (cudaStream_t)stream;
  auto copy = [&](const ktiler_host_copy& c, bool h2d) -> ktiler_status {
    if (c.buf_id < 0 || c.buf_id >= (int32_t)p->g.bufs.size()) return fail(KTILER_E_INVALID, "host copy buffer id out of range");
    const kt::Buffer& b = p->g.bufs[c.buf_id];
    int64_t f0 = c.frame0, nf = c.frames ? c.frames : b.d.frames - f0;
    if (f0 < 0 || f0 + nf > b.d.frames || !c.host) return fail(KTILER_E_INVALID, "host copy frame range");
    if (b.d.ring_frames) return fail(KTILER_E_INVALID, "host copies of a ring buffer (its frames are overwritten)");
    const int64_t rowb = b.d.width * b.d.elem_bytes;
    for (int64_t z = f0; z < f0 + nf; ++z) {
      char* dev = (char*)b.d.base + z * b.d.frame_stride_bytes;
      char* host = (char*)c.host + (z - f0) * rowb * b.d.height;
      cudaError_t e = h2d ? cudaMemcpy2DAsync(dev, b.d.pitch_bytes, host, rowb, rowb, b.d.height, cudaMemcpyHostToDevice, st)
                          : cudaMemcpy2DAsync(host, rowb, dev, b.d.pitch_bytes, rowb, b.d.height, cudaMemcpyDeviceToHost, st);
      if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy2DAsync");
    }
    return KTILER_OK;
  };
  for (int i = 0; i < nin; ++i) {
    ktiler_status s = copy(in[i], true);
    if (s) return s;
  }
  ktiler_status s = ktiler_execute(p, stream);
  if (s) return s;
  for (int i = 0; i < nout; ++i) {
    s = copy(outc[i], false);
    if (s) return s;
  }
  return KTILER_OK;
}

ktiler_status ktiler_plan_num_clusters(ktiler_plan_t p, int32_t* n) {
  if (!p || !n) return fail(KTILER_E_INVALID, "NULL argument");
  *n = (int32_t)p->s.clusters.size();
  return KTILER_OK;
}

ktiler_status ktiler_plan_get_cluster(ktiler_plan_t p, int32_t i, int32_t* nodes, int32_t cap, int32_t* n_nodes,
                                      double* cost_ms) {
  if (!p || !n_nodes) return fail(KTILER_E_INVALID, "NULL argument");
  if (i < 0 || i >= (int32_t)p->s.clusters.size()) return fail(KTILER_E_INVALID, "cluster index out of range");
  const std::vector<int>& c = p->s.clusters[i];
  *n_nodes = (int32_t)c.size();
  if (nodes)
    for (int32_t k = 0; k < cap && k < (int32_t)c.size(); ++k) nodes[k] = c[k];
  if (cost_ms) *cost_ms = p->s.cluster_cost[i];
  return KTILER_OK;
}

ktiler_status ktiler_calibrate(ktiler_graph_t gh, int32_t node, int32_t npts, const int64_t* nb, int32_t reps,
                               double* ms_cold, double* ms_hot) {
  if (!gh || !nb || !ms_cold || !ms_hot || npts < 1 || reps < 1) return fail(KTILER_E_INVALID, "bad argument");
  kt::Graph* G = kt::graph_of(gh);
  ktiler_status s = G->finalize();
  if (s) return s;
  if (node < 0 || node >= (int)G->nodes.size()) return fail(KTILER_E_INVALID, "node out of range");
  if (G->nodes[node].op == KTILER_OP_CUSTOM) return fail(KTILER_E_UNSUPPORTED, "calibration runs built-in ops only");
  ktiler_plan_s P;  // launch context (STREAM semantics)
  P.g = *G;
  P.pol.exec_mode = KTILER_EXEC_STREAM;
  cudaError_t e = cudaGetDevice(&P.device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
  int l2 = 0;
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, P.device);
  const size_t flush_bytes = (size_t)std::max(l2, 1 << 20) * 2;
  void* flush = nullptr;
  if ((e = cudaMalloc(&flush, flush_bytes)) != cudaSuccess) return cuda_fail(e, "cudaMalloc (L2 flush)");
  cudaStream_t st = nullptr;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  const kt::Graph& g = P.g;
  const kt::Node& n = g.nodes[node];
  // the first k blocks of a node in (x, y, z) order as at most 3 rects
  auto first_rects = [](const kt::Node& v, int64_t k) {
    std::vector<kt::Rect6> r;
    const int64_t gx = v.gx(), gy = v.gy(), per = gx * gy;
    const int64_t fz = k / per, rem = k % per, rows = rem / gx, tail = rem % gx;
    if (fz) r.push_back({0, 0, 0, (int32_t)gx, (int32_t)gy, (int32_t)fz});
    if (rows) r.push_back({0, 0, (int32_t)fz, (int32_t)gx, (int32_t)rows, (int32_t)fz + 1});
    if (tail) r.push_back({0, (int32_t)rows, (int32_t)fz, (int32_t)tail, (int32_t)rows + 1, (int32_t)fz + 1});
    return r;
  };
  // device-side spans (first CTA start -> last CTA end) through the tracer
  const int64_t tper = 1 << 10, tcap = tper * TRACE_SHARDS;  // per-SM shards (TraceBuf)
  void* tmem = nullptr;
  if ((e = cudaMalloc(&tmem, (size_t)tcap * sizeof(ktiler_trace_record) + TRACE_SHARDS * 8)) != cudaSuccess)
    return cuda_fail(e, "cudaMalloc (calibration trace)");
  TraceBuf tb{(ktiler_trace_record*)tmem, (unsigned long long*)((char*)tmem + (size_t)tcap * sizeof(ktiler_trace_record)),
              tper};
  cudaMemset(tb.n, 0, TRACE_SHARDS * sizeof(unsigned long long));
  std::vector<ktiler_trace_record> rec;
  auto read_span = [&](uint64_t id, uint64_t* t0, uint64_t* t1) -> bool {  // after a sync
    unsigned long long cnt[TRACE_SHARDS];
    cudaMemcpy(cnt, tb.n, sizeof(cnt), cudaMemcpyDeviceToHost);
    rec.clear();
    for (int sh = 0; sh < TRACE_SHARDS; ++sh) {
      const int64_t k = std::min<int64_t>((int64_t)cnt[sh], tper);
      const size_t at = rec.size();
      rec.resize(at + (size_t)k);
      if (k) cudaMemcpy(rec.data() + at, tb.rec + sh * tper, (size_t)k * sizeof(ktiler_trace_record), cudaMemcpyDeviceToHost);
    }
    *t0 = ~0ull;
    *t1 = 0;
    for (auto& r : rec)
      if (r.kind == 0 && r.id == id) {
        *t0 = std::min(*t0, r.t0_ns);
        *t1 = std::max(*t1, r.t1_ns);
      }
    return *t1 > 0;
  };
  auto launch_rects = [&](int v, const std::vector<kt::Rect6>& rects, int64_t trace_id, int times = 1) -> ktiler_status {
    kt::SubKernel sk;
    sk.node = v;
    sk.rects = rects;
    for (auto& q : rects) sk.nblocks += q.count();
    ktiler_plan_s Q;
    Q.g = g;
    Q.pol.exec_mode = KTILER_EXEC_STREAM;
    Q.device = P.device;
    Q.s.subs.push_back(sk);
    Q.s.discards.resize(1);
    Q.s.nfrag = 1;
    build_launches(&Q);
    for (auto& L : Q.launches) {
      if (L.node >= 0 && !L.n->scalar && L.kp.stage_bytes) {
        L.n = &Q.g.nodes[L.node];
        L.kp.use_tmap = make_tmap(Q.g, *L.n, &L.kp.tmap, &L.kp.box_bytes);
      }
      if (trace_id >= 0) {
        L.kp.tb = tb;
        L.kp.lid = trace_id;
      }
    }
    ktiler_status r = enqueue(&Q, st);
    for (int k = 1; k < times && !r; ++k) {  // back to back: no host work in between
      for (auto& L : Q.launches) ++L.kp.lid;
      r = enqueue(&Q, st);
    }
    return r;
  };
  std::vector<double> ts;
  ktiler_status rs = KTILER_OK;
  // inter-launch gap of back-to-back launches (last CTA end -> next first CTA start):
  // every sub-kernel of a replayed schedule pays it once ("inter-launch gap")
  double gap_ms = 0;
  {
    const std::vector<kt::Rect6> one = first_rects(n, std::min<int64_t>(n.nblocks, n.gx()));
    std::vector<double> gaps;
    for (int r = 0; r < reps + 1 && !rs; ++r) {
      cudaMemsetAsync(tb.n, 0, TRACE_SHARDS * sizeof(unsigned long long), st);
      rs = launch_rects(node, one, 2, 2);  // trace ids 2 and 3
      cudaStreamSynchronize(st);
      uint64_t a0, a1, b0, b1;
      if (r && read_span(2, &a0, &a1) && read_span(3, &b0, &b1) && b0 > a1) gaps.push_back((double)(b0 - a1) * 1e-6);
    }
    std::sort(gaps.begin(), gaps.end());
    gap_ms = gaps.empty() ? 0 : gaps[gaps.size() / 2];
  }
  for (int k = 0; k < npts && !rs; ++k) {
    const int64_t m = std::min<int64_t>(std::max<int64_t>(1, nb[k]), n.nblocks);
    const std::vector<kt::Rect6> rects = first_rects(n, m);
    // producer blocks the first m blocks read: per channel, the bounding block range
    std::vector<std::pair<int, std::vector<kt::Rect6>>> prod;
    for (const kt::Chan& c : g.in_ch[node]) {
      std::vector<kt::Rect6> pr;
      for (auto& q : rects) {
        kt::BRange a = g.producers(c, q.x0, q.y0), b = g.producers(c, q.x1 - 1, q.y1 - 1);
        pr.push_back({(int32_t)a.x0, (int32_t)a.y0, q.z0, (int32_t)b.x1, (int32_t)b.y1, q.z1});
      }
      prod.push_back({c.u, pr});
    }
    for (int hot = 0; hot < 2 && !rs; ++hot) {
      ts.clear();
      for (int r = 0; r < reps + 1 && !rs; ++r) {  // +1: untimed warm-up
        cudaMemsetAsync(flush, r & 0xFF, flush_bytes, st);
        if (hot)
          for (auto& pp : prod)
            if (!rs) rs = launch_rects(pp.first, pp.second, -1);
        cudaMemsetAsync(tb.n, 0, TRACE_SHARDS * sizeof(unsigned long long), st);
        if (!rs) rs = launch_rects(node, rects, 1);
        cudaStreamSynchronize(st);
        uint64_t t0, t1;
        if (r && read_span(1, &t0, &t1)) ts.push_back((double)(t1 - t0) * 1e-6 + gap_ms);
      }
      std::sort(ts.begin(), ts.end());
      (hot ? ms_hot : ms_cold)[k] = ts.empty() ? 0 : ts[ts.size() / 2];
    }
  }
  cudaFree(tmem);
  cudaStreamDestroy(st);
  cudaFree(flush);
  if (rs) return rs;
  if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e, "calibration");
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_discover_footprint(ktiler_graph_t gh, int32_t node, int32_t bx, int32_t by, int32_t bz,
                                        int32_t trials, uint64_t seed, ktiler_footprint_rec* out, int32_t cap,
                                        int32_t* n_out) {
  if (!gh || !n_out || trials < 1) return fail(KTILER_E_INVALID, "bad argument");
  kt::Graph* G = kt::graph_of(gh);
  ktiler_status s = G->finalize();
  if (s) return s;
  if (node < 0 || node >= (int)G->nodes.size()) return fail(KTILER_E_INVALID, "node out of range");
  const kt::Node& nd = G->nodes[node];
  if (bx < 0 || by < 0 || bz < 0 || bx >= nd.gx() || by >= nd.gy() || bz >= nd.gz())
    return fail(KTILER_E_INVALID, "block out of the node's grid");
  // the candidate space: every byte of every buffer (nothing of the declared accesses is used)
  const int nb = (int)G->bufs.size();
  std::vector<int64_t> off(nb + 1, 0);
  for (int b = 0; b < nb; ++b) {
    if (G->bufs[b].addr % 128) return fail(KTILER_E_INVALID, "footprint discovery needs 128-B aligned buffers");
    off[b + 1] = off[b] + ((G->bufs[b].span + 127) & ~(int64_t)127);
  }
  const int64_t total = off[nb];
  if (total > ((int64_t)1 << 30)) return fail(KTILER_E_UNSUPPORTED, "footprint discovery: graph buffers exceed 1 GiB");
  ktiler_plan_s P;  // launch context (STREAM semantics)
  P.g = *G;
  P.pol.exec_mode = KTILER_EXEC_STREAM;
  cudaError_t e = cudaGetDevice(&P.device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
  uint8_t *snap = nullptr, *ref = nullptr, *wr = nullptr;
  unsigned int* flag = nullptr;
  if ((e = cudaMalloc(&snap, (size_t)total)) != cudaSuccess || (e = cudaMalloc(&ref, (size_t)total)) != cudaSuccess ||
      (e = cudaMalloc(&wr, (size_t)total)) != cudaSuccess || (e = cudaMalloc(&flag, 4)) != cudaSuccess) {
    cudaFree(snap); cudaFree(ref); cudaFree(wr);
    return cuda_fail(e, "cudaMalloc (footprint discovery)");
  }
  cudaStream_t st = nullptr;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  auto bufp = [&](int b) { return (uint8_t*)G->bufs[b].d.base; };
  auto span = [&](int b) { return G->bufs[b].span; };
  auto copy_all = [&](uint8_t* dst, bool to_buffers) {
    for (int b = 0; b < nb; ++b)
      if (to_buffers) cudaMemcpyAsync(bufp(b), dst + off[b], (size_t)span(b), cudaMemcpyDeviceToDevice, st);
      else cudaMemcpyAsync(dst + off[b], bufp(b), (size_t)span(b), cudaMemcpyDeviceToDevice, st);
  };
  // one launch of the single block, through the same launcher as every schedule
  kt::SubKernel sk;
  sk.node = node;
  sk.rects.push_back({bx, by, bz, bx + 1, by + 1, bz + 1});
  sk.nblocks = 1;
  P.s.subs.push_back(sk);
  P.s.discards.resize(1);
  P.s.nfrag = 1;
  build_launches(&P);
  for (auto& L : P.launches)
    if (L.node >= 0 && L.n->op != KTILER_OP_CUSTOM && !L.n->scalar && L.kp.stage_bytes) {
      L.n = &P.g.nodes[L.node];
      L.kp.use_tmap = make_tmap(P.g, *L.n, &L.kp.tmap, &L.kp.box_bytes);
    }
  ktiler_status rs = KTILER_OK;
  auto run_block = [&]() { if (!rs) rs = enqueue(&P, st); };
  // 1. writes: union over `trials` independent fills of the bytes the block changed
  cudaMemsetAsync(wr, 0, (size_t)total, st);
  for (int t = 0; t < trials && !rs; ++t) {
    for (int b = 0; b < nb; ++b)
      disc_fill_kernel<<<256, 256, 0, st>>>(bufp(b), span(b), seed * 0x9E3779B97F4A7C15ull + (uint64_t)t * 1000003u + (uint64_t)b);
    copy_all(snap, false);
    run_block();
    for (int b = 0; b < nb && !rs; ++b) disc_diff_kernel<<<256, 256, 0, st>>>(bufp(b), snap + off[b], wr + off[b], span(b));
  }
  // 2. reads: reference = trial-0 fill (snap) and its output (ref); probe(lines [a, b) of the
  //    concatenated line space) = restore, perturb those lines, run, compare on the written bytes
  for (int b = 0; b < nb; ++b)
    disc_fill_kernel<<<256, 256, 0, st>>>(bufp(b), span(b), seed * 0x9E3779B97F4A7C15ull + (uint64_t)b);
  copy_all(snap, false);
  run_block();
  copy_all(ref, false);
  std::vector<int64_t> loff(nb + 1, 0);
  for (int b = 0; b < nb; ++b) loff[b + 1] = loff[b] + (off[b + 1] - off[b]) / 128;
  uint64_t probe_salt = seed ^ 0xD1B54A32D192ED03ull;
  // one perturbation of lines [la, lb): does any written byte change?
  auto probe1 = [&](int64_t la, int64_t lb) -> bool {
    copy_all(snap, true);
    for (int b = 0; b < nb; ++b) {
      const int64_t a = std::max(la, loff[b]), c = std::min(lb, loff[b + 1]);
      if (a >= c) continue;
      const int64_t ba = (a - loff[b]) * 128, bb = std::min((c - loff[b]) * 128, span(b));
      if (ba < bb) disc_perturb_kernel<<<64, 256, 0, st>>>(bufp(b), ba, bb, probe_salt);
    }
    probe_salt = probe_salt * 6364136223846793005ull + 1442695040888963407ull;
    run_block();
    cudaMemsetAsync(flag, 0, 4, st);
    for (int b = 0; b < nb; ++b)
      disc_cmp_kernel<<<128, 256, 0, st>>>(bufp(b), ref + off[b], wr + off[b], span(b), flag);
    unsigned int h = 0;
    cudaMemcpyAsync(&h, flag, 4, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
    return h != 0;
  };
  // a set is independent only if `trials` independent random perturbations all leave the
  // written bytes unchanged (a single one can cancel out through the kernel's arithmetic,
  // e.g. opposite changes of two taps of a filter)
  auto probe = [&](int64_t la, int64_t lb) -> bool {
    for (int t = 0; t < std::max(2, trials); ++t)
      if (probe1(la, lb)) return true;
    return false;
  };
  std::vector<int64_t> read_lines;
  std::vector<std::pair<int64_t, int64_t>> stack{{0, loff[nb]}};
  while (!stack.empty() && !rs) {
    auto [a, b] = stack.back();
    stack.pop_back();
    if (!probe(a, b)) continue;
    if (b - a == 1) {
      read_lines.push_back(a);
    } else {
      const int64_t m = a + (b - a) / 2;
      stack.push_back({m, b});
      stack.push_back({a, m});
    }
  }
  std::vector<uint8_t> hw((size_t)total);
  if (!rs) {
    cudaMemcpyAsync(hw.data(), wr, (size_t)total, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
  }
  e = cudaGetLastError();
  cudaFree(snap); cudaFree(ref); cudaFree(wr); cudaFree(flag);
  cudaStreamDestroy(st);
  if (rs) return rs;
  if (e != cudaSuccess) return cuda_fail(e, "footprint discovery");
  // records: runs of written bytes, runs of read lines (as bytes), per buffer
  std::vector<ktiler_footprint_rec> rec;
  for (int b = 0; b < nb; ++b)
    for (int64_t i = 0; i < span(b);) {
      if (!hw[(size_t)(off[b] + i)]) { ++i; continue; }
      int64_t j = i;
      while (j < span(b) && hw[(size_t)(off[b] + j)]) ++j;
      rec.push_back({b, KTILER_WRITE, i, j});
      i = j;
    }
  std::sort(read_lines.begin(), read_lines.end());
  for (size_t i = 0; i < read_lines.size();) {
    size_t j = i + 1;
    while (j < read_lines.size() && read_lines[j] == read_lines[j - 1] + 1) ++j;
    int b = 0;
    while (read_lines[i] >= loff[b + 1]) ++b;
    const int64_t first = (read_lines[i] - loff[b]) * 128;
    const int64_t last = std::min((read_lines[j - 1] - loff[b] + 1) * 128, span(b));
    // a run never crosses buffers: split where it does
    int64_t k = (int64_t)i;
    while (k < (int64_t)j) {
      int bb = 0;
      while (read_lines[k] >= loff[bb + 1]) ++bb;
      int64_t e2 = k;
      while (e2 + 1 < (int64_t)j && read_lines[e2 + 1] < loff[bb + 1]) ++e2;
      rec.push_back({bb, KTILER_READ, (read_lines[k] - loff[bb]) * 128,
                     std::min((read_lines[e2] - loff[bb] + 1) * 128, span(bb))});
      k = e2 + 1;
    }
    (void)first; (void)last;
    i = j;
  }
  *n_out = (int32_t)rec.size();
  if (out)
    for (int32_t k = 0; k < cap && k < (int32_t)rec.size(); ++k) out[k] = rec[k];
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_selftest(int32_t which, int64_t* failures) {
  if (!failures) return fail(KTILER_E_INVALID, "NULL argument");
  if (which != KTILER_SELFTEST_SQRT) return fail(KTILER_E_INVALID, "unknown self-test");
  unsigned long long* d = nullptr;
  cudaError_t e = cudaMalloc(&d, sizeof(*d));
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (selftest)");
  cudaMemset(d, 0, sizeof(*d));
  selftest_sqrt_kernel<<<1184, 256>>>(2u * 1020u * 1020u, d);
  unsigned long long h = 0;
  e = cudaMemcpy(&h, d, sizeof(h), cudaMemcpyDeviceToHost);
  cudaFree(d);
  if (e != cudaSuccess) return cuda_fail(e, "selftest");
  *failures = (int64_t)h;
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_trace_enable(ktiler_plan_t p, int64_t capacity) {
  if (!p || capacity <= 0) return fail(KTILER_E_INVALID, "NULL plan or capacity <= 0");
  if (p->executed || p->tb.rec) return fail(KTILER_E_STATE, "ktiler_trace_enable must precede the first execute");
  void* d = nullptr;
  // capacity records in TRACE_SHARDS per-SM shards (rounded up), then the shard counters
  const int64_t per = (capacity + TRACE_SHARDS - 1) / TRACE_SHARDS;
  const size_t rec_bytes = (size_t)per * TRACE_SHARDS * sizeof(ktiler_trace_record);
  const size_t bytes = rec_bytes + TRACE_SHARDS * sizeof(unsigned long long);
  cudaError_t e = cudaMalloc(&d, bytes);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (trace)");
  if ((e = cudaMemset(d, 0, bytes)) != cudaSuccess) return cuda_fail(e, "cudaMemset (trace)");
  p->tb.rec = (ktiler_trace_record*)d;
  p->tb.n = (unsigned long long*)((char*)d + rec_bytes);
  p->tb.cap = per;
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_trace_read(ktiler_plan_t p, ktiler_trace_record* out, int64_t cap, int64_t* n) {
  if (!p || !n) return fail(KTILER_E_INVALID, "NULL argument");
  if (!p->tb.rec) return fail(KTILER_E_STATE, "tracing not enabled");
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceSynchronize");
  unsigned long long cnt[TRACE_SHARDS];
  if ((e = cudaMemcpy(cnt, p->tb.n, sizeof(cnt), cudaMemcpyDeviceToHost)) != cudaSuccess) return cuda_fail(e, "cudaMemcpy");
  int64_t total = 0;
  for (int sh = 0; sh < TRACE_SHARDS; ++sh) total += (int64_t)cnt[sh];
  *n = total;
  if (out && cap > 0) {
    int64_t k = 0;  // gather the shards' written records, shard by shard
    for (int sh = 0; sh < TRACE_SHARDS && k < cap; ++sh) {
      const int64_t m = std::min<int64_t>({(int64_t)cnt[sh], p->tb.cap, cap - k});
      if (m > 0 && (e = cudaMemcpy(out + k, p->tb.rec + (int64_t)sh * p->tb.cap, (size_t)m * sizeof(ktiler_trace_record),
                                   cudaMemcpyDeviceToHost)) != cudaSuccess)
        return cuda_fail(e, "cudaMemcpy");
      k += m;
    }
    if ((e = cudaMemset(p->tb.n, 0, sizeof(cnt))) != cudaSuccess) return cuda_fail(e, "cudaMemset");
  }
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_plan_get_launch(ktiler_plan_t p, int64_t i, int32_t* sub, int32_t* node, int64_t* tiles) {
  if (!p) return fail(KTILER_E_INVALID, "NULL plan");
  const int64_t nl = (int64_t)p->launches.size(), nd = (int64_t)p->dag_disc.size();
  if (i < 0 || i >= nl + nd) return fail(KTILER_E_INVALID, "launch index out of range");
  const Launch& L = i < nl ? p->launches[i] : p->dag_disc[i - nl];
  if (sub) *sub = L.node >= 0 ? L.sub : -1;
  if (node) *node = L.node;
  if (tiles) *tiles = L.node >= 0 ? L.blocks : 0;
  return KTILER_OK;
}

}  // extern "C"
