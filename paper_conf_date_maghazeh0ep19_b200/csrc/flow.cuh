// KTILER_EXEC_FLOW: the persistent executor driven by per-tile dependency flags
// (BASELINE north_star "a persistent-kernel variant driven by per-tile dependency flags").
//
// The schedule (a total order of sub-kernels) is replayed at tile
// granularity by ONE cooperative launch of K CTAs per SM.  Every CTA serves one *role*
// (a set of the graph's kernels, ktiler_plan_set_flow_roles), chosen from its slot on its
// SM (%smid), so each SM hosts the same mix of roles and each CTA keeps running the same
// kernel body (its instruction stream and staging layout stay warm).  A role's CTAs claim
// the role's tiles one at a time, in the role's ticket order, from one atomic counter.
//
// Dependencies are the paper's block-level RAW dependencies: before a
// tile is staged, the producer warp waits (ld.acquire.gpu) until the epoch flag of every
// producer tile whose output rect meets the tile's read footprint (closed form of the
// affine maps) carries this execute's epoch; the compute warps publish
// their own tile's flag (st.release.gpu after a CTA-scope barrier) when it is written.
// A consumer tile therefore waits only for the producer tiles that cover it, never for a
// whole sub-kernel.
//
// The L2 budget of Alg. 2 becomes a run-ahead window: a tile of a source
// kernel in fragment f may start only once the leaf kernels' tiles of fragments <= f - W
// are complete (one leaf-completion counter), so the live intermediates stay within W
// fragments.
//
// Deadlock freedom: every role's ticket list is the restriction of ONE global order, the
// software-pipelined order over fragments (the sub-kernel of fragment f at node depth d in
// step f + d*skew, deepest first; DESIGN A37) — a dependency-respecting total order
// in which every producer tile and every window dependency lies strictly
// earlier (the host enforces W > depth_max * skew).  A CTA processes its claims in order
// and compute warps never wait on other CTAs, so the globally earliest unfinished tile is
// always claimed by a CTA that is working on it; the cooperative launch guarantees every
// role's CTAs are co-resident.  A bounded spin (watchdog) traps instead of hanging if that
// invariant were ever broken.
#pragma once

#include "kernels.cuh"
#include "ktiler.h"

namespace ktflow {

using ktd::DBuf;

constexpr int FSLOTS_MAX = 8;
constexpr int FMAX_NODES = 1024;
constexpr int FMAX_ROLES = 16;
constexpr int FMAX_SLOTS = 16;

struct FNode {
  CUtensorMap tmap;  // input tile map (tensor TMA)
  DBuf in, out;
  DBuf aux;          // KTILER_OP_JACOBI: the coefficient buffer (a graph input)
  float taps[9];     // KTILER_OP_GAUSS_F32: f32 weights, taps[k + radius]
  int32_t radius;
  int64_t flag0;     // this node's first tile flag
  int64_t pflag0;    // its producer node's first tile flag
  uint32_t box_bytes;
  int32_t op, tw, th, in_stream, cdisc, leaf;
  float T;
  int32_t gx, gy;    // this node's grid (flag index = (bz * gy + by) * gx + bx)
  int32_t pgx, pgy;  // producer's grid (pgx == 0: reads a graph input, nothing to wait on)
  int32_t rax, ray, rox, roy, rhl, rhr, rht, rhb;  // read footprint (affine map)
  int32_t wax, way;  // producer's write footprint
};

// device timeline (ktiler_trace_enable): kinds 5 = a tile's claim -> TMA issue (producer
// warp), 6 = its compute (compute thread 0: slot full -> own stores done), 7 = its flag
// published (t0 = t1); id = the ticket
struct FTrace {
  ktiler_trace_record* rec;
  unsigned long long* n;
  int64_t cap;
};
constexpr int FL_TRACE_SHARDS = 256;  // == exec.cu TRACE_SHARDS
__device__ __forceinline__ uint64_t fl_timer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void fl_trace(const FTrace& tb, uint64_t id, uint32_t kind, uint64_t t0, uint64_t t1) {
  // the plan's per-SM sharded trace buffer (exec.cu TraceBuf): FL_TRACE_SHARDS counters,
  // cap records per shard
  uint32_t sm;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
  // shard by a hash of (record id, CTA, SM): small launches fill the low SM ids with
  // low CTA indices first, so SM or CTA alone would crowd a few shards
  const uint32_t sh =
      ((blockIdx.x * 0x9E3779B9u) ^ (sm * 0x85EBCA6Bu) ^ ((uint32_t)id * 0xC2B2AE35u)) >> 24 & (FL_TRACE_SHARDS - 1);
  const unsigned long long k = atomicAdd(tb.n + sh, 1ull);
  if ((int64_t)k < tb.cap) tb.rec[(int64_t)sh * tb.cap + (int64_t)k] = ktiler_trace_record{id, sm, kind, t0, t1};
}

struct FCtrl {
  unsigned int epoch, done, leaf_done, pad;
};

struct FParams {
  const FNode* nodes;
  const uint64_t* tickets;    // role lists, contiguous
  const int64_t* role_off;    // [nroles + 1]
  const int32_t* slot_role;   // [nslots_sm]
  unsigned int* claim;        // [nroles] next unclaimed ticket of each role
  unsigned int* smslot;       // [256] CTAs that have taken a slot on each SM
  unsigned int* flags;        // per tile, all nodes
  FCtrl* ctrl;
  int32_t role_stage[FMAX_ROLES];   // bytes of one ring slot of each role (its largest staged tile)
  int32_t role_nslots[FMAX_ROLES];  // ring depth of each role (the CTA's shared memory / slot)
  int32_t nslots_sm;          // CTAs (slots) per SM
  int32_t nroles;
  int32_t nnodes;
  uint64_t spin_limit;        // watchdog: polls before __trap (0 = none)
  int32_t batch;              // tickets per claim (1..32)
  int32_t pending;            // claimed, unstaged tickets a producer warp may hold (batch..32)
  FTrace tb;                  // rec == NULL: tracing off
};

// Ticket: node (10) | window (22: leaf tiles that must be complete first) | bz (8) |
// by (12) | bx (12).
__host__ __device__ inline uint64_t flow_ticket(uint64_t node, uint64_t wait, uint64_t bx, uint64_t by, uint64_t bz) {
  return (node << 54) | (wait << 32) | (bz << 24) | (by << 12) | bx;
}
constexpr uint64_t FLOW_WAIT_MAX = (1ull << 22) - 1;
constexpr int FLOW_BZ_MAX = 255, FLOW_BXY_MAX = 4095;
__host__ __device__ __forceinline__ int fl_node(uint64_t d) { return (int)(d >> 54); }
__host__ __device__ __forceinline__ unsigned fl_waitv(uint64_t d) { return (unsigned)((d >> 32) & FLOW_WAIT_MAX); }
__host__ __device__ __forceinline__ int fl_bx(uint64_t d) { return (int)(d & 0xFFF); }
__host__ __device__ __forceinline__ int fl_by(uint64_t d) { return (int)((d >> 12) & 0xFFF); }
__host__ __device__ __forceinline__ int fl_bz(uint64_t d) { return (int)((d >> 24) & 0xFF); }
constexpr uint64_t FLOW_STOP = ~0ull;

__device__ __forceinline__ unsigned int fl_acquire(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned int fl_relaxed(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fl_release(unsigned int* p, unsigned int v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void fl_red_release(unsigned int* p, unsigned int v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// generic-proxy writes (other SMs' tile stores, acquired through a flag) before this
// thread's async-proxy (TMA) reads of global memory
__device__ __forceinline__ void fence_proxy_async_all() { asm volatile("fence.proxy.async;" ::: "memory"); }
__device__ __forceinline__ void fl_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void fl_arrive(uint64_t* m) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ktd::smem_u32(m)) : "memory");
}

// Watchdog poll: sleeps between probes; traps (kernel error, not a hang) after spin_limit
// probes — a dependency that can never be satisfied is a schedule bug.
__device__ __forceinline__ void fl_spin(uint64_t& n, uint64_t limit) {
  __nanosleep(64);
  if (limit && ++n > limit) __trap();
}

__device__ __forceinline__ ktd::Tile flow_tile(const FNode& nd, uint64_t d) {
  const int bx = fl_bx(d), by = fl_by(d), bz = fl_bz(d);
  ktd::Tile t;
  t.z = bz;
  t.x0 = (int64_t)nd.tw * bx;
  t.y0 = (int64_t)nd.th * by;
  t.x1 = min(t.x0 + nd.tw, nd.out.W);
  t.y1 = min(t.y0 + nd.th, nd.out.H);
  t.fw = nd.tw;
  t.pad = (bz * nd.gy + by) * nd.gx + bx;  // flag index within the node
  return t;
}

// Producer tile range of tile (bx, by) of node nd: [px0, px1) x [py0, py1) of its producer.
struct PRange {
  int px0, py0, pw, n;
};
__device__ __forceinline__ PRange flow_prange(const FNode& nd, uint64_t d) {
  const int bx = fl_bx(d), by = fl_by(d);
  const int rx0 = max(0, nd.rax * bx + nd.rox - nd.rhl), rx1 = min((int)nd.in.W, nd.rax * (bx + 1) + nd.rox + nd.rhr);
  const int ry0 = max(0, nd.ray * by + nd.roy - nd.rht), ry1 = min((int)nd.in.H, nd.ray * (by + 1) + nd.roy + nd.rhb);
  const int px0 = rx0 / nd.wax, px1 = min(nd.pgx, (rx1 + nd.wax - 1) / nd.wax);
  const int py0 = ry0 / nd.way, py1 = min(nd.pgy, (ry1 + nd.way - 1) / nd.way);
  PRange r;
  r.px0 = px0;
  r.py0 = py0;
  r.pw = max(0, px1 - px0);
  r.n = nd.pgx ? r.pw * max(0, py1 - py0) : 0;
  return r;
}

// Producer warp, non-blocking: which of the claimed tiles (ticket j held by lane j; bit j of
// `left` = still to stage) are ready — every producer tile covering its read footprint has published `epoch`
// (one round of acquire loads over all (tile, flag) pairs, spread over the lanes) and, for
// a source tile, the window's leaf tiles are complete.  Returns a bit mask (bit j = tile j).
__device__ __forceinline__ unsigned flow_ready(const FParams& p, uint64_t mine, unsigned left, unsigned epoch,
                                               int lane) {
  unsigned bad = 0;
  // window (source tiles): one load, compared with every pending tile's requirement
  const unsigned wait = ((left >> lane) & 1u) ? fl_waitv(mine) : 0u;
  if (__any_sync(0xFFFFFFFFu, wait != 0u)) {
    unsigned done = 0;
    if (lane == 0) done = fl_relaxed(&p.ctrl->leaf_done);
    done = __shfl_sync(0xFFFFFFFFu, done, 0);
    if (wait && (int)(done - wait) < 0) bad |= 1u << lane;
  }
  // producer flags: tile j's flags are pairs (j, i < n_j); lane l probes pairs l, l+32, ...
  for (unsigned m = left; m; m &= m - 1) {
    const int j = __ffs(m) - 1;
    const uint64_t d = __shfl_sync(0xFFFFFFFFu, mine, j);
    const FNode& nd = p.nodes[fl_node(d)];
    const PRange r = flow_prange(nd, d);
    const int bz = fl_bz(d);
    for (int i = lane; i < r.n; i += 32) {
      const int dy = i / r.pw;
      const unsigned int* f = p.flags + nd.pflag0 + ((int64_t)bz * nd.pgy + r.py0 + dy) * nd.pgx + r.px0 + (i - dy * r.pw);
      if (fl_relaxed(f) != epoch) bad |= 1u << j;  // relaxed probes overlap; one fence below
    }
  }
  bad = __reduce_or_sync(0xFFFFFFFFu, bad);
  // acquire: the flags observed above synchronize with their publishers' fence + store
  // (fence-based release/acquire, PTX memory model); __syncwarp then orders lane 0's TMA
  // issue after every lane's fence
  asm volatile("fence.acq_rel.gpu;" ::: "memory");
  __syncwarp();
  return ~bad;
}

// KTILER_PF_CONSUMER_DISCARD in FLOW (DESIGN A44): the staged input lines of a tile whose
// node is the buffer's only reader, read without halo (down2: 2 B, thresh: 4 B per output
// pixel along x), leave L2 without write-back.
__device__ __forceinline__ void flow_consumer_discard(const FNode& nd, const ktd::Tile& t, int nt, int tid) {
  const int64_t eb = nd.op == 2 ? 2 : 4;
  const int64_t y0 = nd.op == 2 ? 2 * t.y0 : t.y0, nrows = nd.op == 2 ? 2 * (t.y1 - t.y0) : t.y1 - t.y0;
  const uint8_t* base = nd.in.p + ktd::zoff(nd.in, t.z);
  const int64_t b0 = eb * t.x0, b1 = eb * t.x1;
  const int64_t first = ((int64_t)(uintptr_t)(base + y0 * nd.in.pitch + b0) + 127) >> 7;
  const int64_t last = ((int64_t)(uintptr_t)(base + y0 * nd.in.pitch + b1)) >> 7;
  if (last <= first) return;
  // same count for every row (128-B pitch); 32-bit index math per line (a 64-bit division
  // per line cost more than the tile's own arithmetic)
  const unsigned per = (unsigned)(last - first), n = per * (unsigned)nrows;
  const bool pow2 = (per & (per - 1)) == 0;
  const int sh = __ffs(per) - 1;
  for (unsigned i = tid; i < n; i += nt) {
    const unsigned r = pow2 ? i >> sh : i / per, l = i - r * per;
    const uint8_t* row = base + (y0 + (int64_t)r) * nd.in.pitch;
    ktd::discard_line(reinterpret_cast<const void*>((((int64_t)(uintptr_t)(row + b0) + 127) >> 7 << 7) + 128 * (int64_t)l));
  }
}

// NW compute warps + 1 producer warp per CTA.
//
// Producer warp: an event loop that never blocks.  It claims batches of `batch` tickets of
// its role, checks their dependencies without waiting (flow_ready) and stages every ready
// tile of the batch — in batch order, skipping tiles that are not ready yet — into the
// next ring slot by TMA as soon as that slot's previous tile has been computed (s_done).
// Out-of-order issue inside a claimed batch keeps deadlock freedom: the globally earliest
// unfinished tile is ready, and its CTA's ring drains without waiting on anyone.
//
// Compute warps: wait for their slot's TMA (s_full), compute, arrive on s_done (release at
// CTA scope after their stores).  Tile k is then published by compute warp k mod NW: its
// lane 0 waits for the tile's s_done phase (acquire), issues a gpu-scope fence and stores
// the epoch flag (fence-based release), so the fence latency rotates over the warps and
// never sits on the producer.  Compute warps never wait on other CTAs.  Named barrier 2 =
// stage_fix among the compute warps.
template <int NW, int MINB>
__global__ void __launch_bounds__(32 * (NW + 1), MINB) flow_kernel(const __grid_constant__ FParams p) {
  constexpr int NC = 32 * NW;
  __shared__ __align__(8) uint64_t s_full[FSLOTS_MAX];
  __shared__ __align__(8) uint64_t s_done[FSLOTS_MAX];
  __shared__ uint64_t s_desc[FSLOTS_MAX];
  __shared__ ktd::Tile s_tile[FSLOTS_MAX];
  __shared__ int32_t s_role;
  __shared__ unsigned int s_epoch;
  extern __shared__ __align__(128) uint8_t fsm[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    const unsigned slot = atomicAdd(p.smslot + (smid & 255), 1u);
    const int r = p.slot_role[slot % (unsigned)p.nslots_sm];
    s_role = r;
    s_epoch = *(volatile unsigned int*)&p.ctrl->epoch;
    for (int s = 0; s < p.role_nslots[r]; ++s) {
      ktd::mbar_init(&s_full[s], 1);
      ktd::mbar_init(&s_done[s], NC);
    }
    ktd::fence_proxy_async();
  }
  __syncthreads();
  const int role = s_role;
  const unsigned epoch = s_epoch;
  const int S = p.role_nslots[role];
  const int64_t stage_bytes = p.role_stage[role];
  if (warp == NW) {
    // ------------------------------ producer warp ------------------------------
    // Lane j holds pending ticket j (claimed, not staged yet; bit j of `left`) and its
    // claim position `pos`.  Batches of `batch` tickets are claimed whenever the pending set
    // has room (at most p.pending), so a CTA whose oldest tickets wait on dependencies
    // still finds ready work further on; ready tickets are staged oldest first.
    const uint64_t* tk = p.tickets + p.role_off[role];
    const unsigned ntk = (unsigned)(p.role_off[role + 1] - p.role_off[role]);
    const unsigned B = (unsigned)p.batch;
    const int cap = p.pending;
    unsigned next = 0;  // lane 0: base of the batch claimed in advance
    if (lane == 0) next = atomicAdd(p.claim + role, B);
    uint64_t mine = FLOW_STOP;
    unsigned pos = 0xFFFFFFFFu;  // claim position of this lane's ticket
    unsigned left = 0, rdy = 0;  // pending tickets; those known ready
    int k_iss = 0;               // tiles staged
    bool claims_done = false;
    uint64_t idle = 0, t_batch = 0;
    auto slot_free = [&](int k) {  // slot of tile k: its previous tile (k - S) computed
      bool f = true;
      if (lane == 0 && k >= S) f = ktd::mbar_test(&s_done[k % S], (unsigned)((k - S) / S) & 1u);
      return __shfl_sync(0xFFFFFFFFu, (int)f, 0) != 0;
    };
    for (;;) {
      bool progress = false;
      // ---- claim while the pending set has room ----
      while (!claims_done && __popc(left) + (int)B <= cap) {
        const unsigned base = __shfl_sync(0xFFFFFFFFu, next, 0);
        if (base >= ntk) {
          claims_done = true;
          break;
        }
        if (lane == 0) next = atomicAdd(p.claim + role, B);
        const int qn = (int)min(B, ntk - base);
        // the i-th free lane (i < qn) takes ticket base + i
        const unsigned freem = ~left;
        const int rank = __popc(freem & ((1u << lane) - 1u));
        if (((freem >> lane) & 1u) && rank < qn) {
          mine = __ldg(tk + base + rank);
          pos = base + rank;
        }
        left |= __ballot_sync(0xFFFFFFFFu, ((freem >> lane) & 1u) && rank < qn);
        if (p.tb.rec) t_batch = fl_timer();
        progress = true;
      }
      if (left) {
        if (slot_free(k_iss)) {
          if ((rdy & left) != left) rdy |= flow_ready(p, mine, left & ~rdy, epoch, lane) & left;
          while (rdy & left) {
            if (!slot_free(k_iss)) break;
            // oldest ready ticket
            const bool cand = ((rdy & left) >> lane) & 1u;
            const unsigned best = __reduce_min_sync(0xFFFFFFFFu, cand ? pos : 0xFFFFFFFFu);
            const int j = __ffs(__ballot_sync(0xFFFFFFFFu, cand && pos == best)) - 1;
            left &= ~(1u << j);
            rdy &= ~(1u << j);
            const uint64_t d = __shfl_sync(0xFFFFFFFFu, mine, j);
            if (lane == 0) {
              const FNode& nd = p.nodes[fl_node(d)];
              const int s = k_iss % S;
              const ktd::Tile tl = flow_tile(nd, d);
              s_tile[s] = tl;
              s_desc[s] = d;
              fence_proxy_async_all();
              ktd::stage_issue_tmap(nd.op, &nd.tmap, nd.box_bytes, nd.in, tl, fsm + s * stage_bytes, &s_full[s],
                                    nd.in_stream != 0);
              if (p.tb.rec) fl_trace(p.tb, d, 5, t_batch, fl_timer());
            }
            ++k_iss;
            progress = true;
          }
        }
      } else if (claims_done) {
        if (slot_free(k_iss)) {  // one STOP for the compute warps, then done
          if (lane == 0) {
            s_desc[k_iss % S] = FLOW_STOP;
            fl_arrive(&s_full[k_iss % S]);
          }
          break;
        }
      }
      __syncwarp();
      if (!progress) {
        fl_spin(idle, p.spin_limit);
      } else {
        idle = 0;
      }
    }
  } else {
    // ------------------------------ compute warps ------------------------------
    for (int k = 0;; ++k) {
      const int s = k % S;
      ktd::mbar_wait(&s_full[s], (unsigned)(k / S) & 1u);
      const uint64_t tc0 = p.tb.rec ? fl_timer() : 0;
      const uint64_t d = s_desc[s];
      if (d == FLOW_STOP) break;
      const FNode& nd = p.nodes[fl_node(d)];
      const ktd::Tile t = s_tile[s];
      const uint8_t* buf = fsm + s * stage_bytes;
      if (nd.cdisc) flow_consumer_discard(nd, t, NC, tid);
      if (ktd::needs_fix(nd.op, nd.in, t)) {
        ktd::stage_fix(nd.op, nd.in, t, const_cast<uint8_t*>(buf), NC, tid, 2);
        fl_bar(1, NC);
      }
      ktd::compute_tile(nd.op, nd.out, t, buf, nd.T, NC, tid, &nd.aux, nd.taps, nd.radius);
      if (p.tb.rec && tid == 0) fl_trace(p.tb, d, 6, tc0, fl_timer());
      fl_arrive(&s_done[s]);  // release (CTA scope) after this thread's tile stores
      if (warp == k % NW) {   // this warp publishes tile k
        if (lane == 0) {
          ktd::mbar_wait(&s_done[s], (unsigned)(k / S) & 1u);  // every compute thread's stores
          asm volatile("fence.acq_rel.gpu;" ::: "memory");        // ... visible at gpu scope
          asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p.flags + nd.flag0 + t.pad), "r"(epoch) : "memory");
          if (nd.leaf) asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(&p.ctrl->leaf_done) : "memory");
          if (p.tb.rec) {
            const uint64_t tn = fl_timer();
            fl_trace(p.tb, d, 7, tn, tn);
          }
        }
        __syncwarp();
      }
    }
  }
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    const unsigned old = atomicAdd(&p.ctrl->done, 1u);
    if (old == gridDim.x - 1) {  // the last CTA: reset the per-execute counters
      for (int r = 0; r < p.nroles; ++r) p.claim[r] = 0;
      for (int i = 0; i < 256; ++i) p.smslot[i] = 0;
      p.ctrl->leaf_done = 0;
      p.ctrl->done = 0;
      __threadfence();
      atomicAdd(&p.ctrl->epoch, 1u);
    }
  }
}

}  // namespace ktflow
