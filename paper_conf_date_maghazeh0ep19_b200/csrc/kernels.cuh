// sm_100a tile bodies of the five built-in kernels (SURVEY §8(a) a7–a11).
//
// Every body computes ONE block's output rect [x0,x1) x [y0,y1) of frame z with nt
// threads (thread tid); the rect is exactly the block's declared WRITE footprint, so the
// planner's dependency analysis and the kernels can never disagree.
//
// Vector variant (B200 geometry) = two phases, so the executors can overlap the memory of
// one tile with the arithmetic of another:
//   staging       the block's input footprint (+ halo) lands in shared memory by ONE
//                 tensor-map TMA (cp.async.bulk.tensor.3d, completion on an mbarrier); a
//                 replicate fix-up (stage_fix) reproduces the image-edge clamp that TMA's
//                 zero fill does not;
//   compute_tile  one work item = 16 output pixels of one row (gray, down2, thresh) or a
//                 16-pixel column strip of rows_per_item rows with a sliding row window in
//                 registers (blur5, sobel3); packed 2x16-bit SIMD arithmetic in 32-bit
//                 registers, byte permutes (PRMT) to unpack/pack, dp2a for the luma dot
//                 product, 128-bit stores (256-bit for the f32 Sobel rows).
// Scalar variant: the paper's Fig. 1 geometry, one thread per pixel.
// Cache policy: the graph input (rgb) is read once -> L2 evict_first; in a tiled plan so
// is every intermediate with a single reader node (its consumer is its last reader,
// DESIGN.md A42); the graph output (mask) is never re-read -> L2 evict_first stores;
// intermediate stores keep the default policy so they stay resident for their consumer
// sub-kernel (the point of KTILER).
// Border: replicate (clamp-to-edge) at image edges only.
#pragma once

#include <cuda.h>  // CUtensorMap

#include <cstdint>

namespace ktd {

struct DBuf {
  uint8_t* p;
  int64_t W, H, pitch, fstride;
  int32_t ring;  // 0, or a WAR-aware ring of `ring` frames: frame z lives in slot z mod ring
  int32_t pad;
};
// byte offset of frame z in b
__host__ __device__ __forceinline__ int64_t zoff(const DBuf& b, int64_t z) {
  return (b.ring ? (int64_t)((uint32_t)z % (uint32_t)b.ring) : z) * b.fstride;
}

// ---------------------------------------------------------------------------------
// memory helpers
// ---------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ uint8_t ld1(const uint8_t* p) { return __ldcg(p); }
__device__ __forceinline__ void st16(void* p, uint4 v) { *reinterpret_cast<uint4*>(p) = v; }
__device__ __forceinline__ void st16_stream(void* p, uint4 v, uint64_t pol) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p), "r"(v.x),
               "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol)
               : "memory");
}
// 32 bytes (8 words, 32-B aligned) in one 256-bit store (sm_100: STG.E.256)
__device__ __forceinline__ void st32(void* p, const uint32_t* v) {
  asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]),
               "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
               : "memory");
}
__device__ __forceinline__ void discard_line(const void* p) {
  asm volatile("discard.global.L2 [%0], 128;" ::"l"(p) : "memory");
}

__device__ __forceinline__ int64_t clampi(int64_t v, int64_t lo, int64_t hi) { return v < lo ? lo : (v > hi ? hi : v); }
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t s) { return __byte_perm(a, b, s); }
__device__ __forceinline__ const uint8_t* row_ptr(const DBuf& b, int64_t z, int64_t y) {
  return b.p + zoff(b, z) + y * b.pitch;
}
__device__ __forceinline__ uint4 lds16(const uint8_t* p) { return *reinterpret_cast<const uint4*>(p); }
__device__ __forceinline__ uint32_t lds4(const uint8_t* p) { return *reinterpret_cast<const uint32_t*>(p); }

struct Tile {
  int64_t z, x0, y0, x1, y1;  // output rect [x0,x1) x [y0,y1) of frame z
  int fw;                     // full tile width (px): fixes the staging row stride, so
  int pad;                    // ragged edge tiles use the same layout as the TMA box
  __device__ int nseg() const { return (int)((x1 - x0 + 15) >> 4); }
  __device__ int fseg() const { return (fw + 15) >> 4; }
  __device__ int rows() const { return (int)(y1 - y0); }
};

// ---------------------------------------------------------------------------------
// scalar (one pixel) definitions: the one-thread-per-pixel variant
// ---------------------------------------------------------------------------------
__device__ __forceinline__ uint8_t gray_px(const uint8_t* s) {
  uint32_t R = s[0], G = s[1], B = s[2];
  return (uint8_t)((19595u * R + 38470u * G + 7471u * B + 32768u) >> 16);
}
__device__ __forceinline__ uint8_t blur_px(const DBuf& in, int64_t z, int64_t y, int64_t x) {
  const int w[5] = {1, 4, 6, 4, 1};
  int32_t s = 0;
#pragma unroll
  for (int i = 0; i < 5; ++i) {
    const uint8_t* r = row_ptr(in, z, clampi(y + i - 2, 0, in.H - 1));
    int32_t h = 0;
#pragma unroll
    for (int j = 0; j < 5; ++j) h += w[j] * (int32_t)ld1(r + clampi(x + j - 2, 0, in.W - 1));
    s += w[i] * h;
  }
  return (uint8_t)((s + 128) >> 8);
}
__device__ __forceinline__ uint8_t down_px(const DBuf& in, int64_t z, int64_t y, int64_t x) {
  const uint8_t* r0 = row_ptr(in, z, 2 * y);
  const uint8_t* r1 = row_ptr(in, z, 2 * y + 1);
  return (uint8_t)(((uint32_t)ld1(r0 + 2 * x) + ld1(r0 + 2 * x + 1) + ld1(r1 + 2 * x) + ld1(r1 + 2 * x + 1) + 2) >> 2);
}
__device__ __forceinline__ float sobel_px(const DBuf& in, int64_t z, int64_t y, int64_t x) {
  const uint8_t* rm = row_ptr(in, z, clampi(y - 1, 0, in.H - 1));
  const uint8_t* r0 = row_ptr(in, z, y);
  const uint8_t* rp = row_ptr(in, z, clampi(y + 1, 0, in.H - 1));
  int64_t xm = clampi(x - 1, 0, in.W - 1), xp = clampi(x + 1, 0, in.W - 1);
  int32_t gx = (ld1(rm + xp) + 2 * ld1(r0 + xp) + ld1(rp + xp)) - (ld1(rm + xm) + 2 * ld1(r0 + xm) + ld1(rp + xm));
  int32_t gy = (ld1(rp + xm) + 2 * ld1(rp + x) + ld1(rp + xp)) - (ld1(rm + xm) + 2 * ld1(rm + x) + ld1(rm + xp));
  return __fsqrt_rn((float)(gx * gx + gy * gy));
}

__device__ void scalar_tile(int op, const DBuf& in, const DBuf& out, const Tile& t, float T, int nt, int tid) {
  const int64_t w = t.x1 - t.x0, n = w * (t.y1 - t.y0);
  for (int64_t i = tid; i < n; i += nt) {
    const int64_t x = t.x0 + i % w, y = t.y0 + i / w;
    uint8_t* d = const_cast<uint8_t*>(row_ptr(out, t.z, y));
    switch (op) {
      case 0: d[x] = gray_px(row_ptr(in, t.z, y) + 3 * x); break;
      case 1: d[x] = blur_px(in, t.z, y, x); break;
      case 2: d[x] = down_px(in, t.z, y, x); break;
      case 3: reinterpret_cast<float*>(d)[x] = sobel_px(in, t.z, y, x); break;
      case 4: d[x] = __ldcg(reinterpret_cast<const float*>(row_ptr(in, t.z, y)) + x) > T ? 255 : 0; break;
    }
  }
}

// ---------------------------------------------------------------------------------
// staging
// ---------------------------------------------------------------------------------

// ---- TMA bulk copies completing on an mbarrier (the Blackwell async proxy) ----
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* m, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(count) : "memory");
}
// make mbarrier inits / generic smem accesses visible to the async proxy
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_arrive_expect(uint64_t* m, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* m) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(m))
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* m, unsigned parity) {
  asm volatile(
      "{\n .reg .pred P;\n KT_WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n @!P bra KT_WAIT_%=;\n}" ::"r"(
          smem_u32(m)),
      "r"(parity)
      : "memory");
}

// non-blocking probe of an mbarrier phase (parity)
__device__ __forceinline__ bool mbar_test(uint64_t* m, unsigned parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred P;\n mbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n selp.u32 %0, 1, 0, P;\n}"
      : "=r"(ok)
      : "r"(smem_u32(m)), "r"(parity)
      : "memory");
  return ok != 0;
}

// Staged window of op's input for tile t: rows [ry0, ry0+nr) (clamped to the image for the
// stencils), byte columns [xb0, xb0 + stride) (negative / beyond-width columns of the
// stencils are filled by stage_fix with the replicate rule).
constexpr int GAUSS_H = 4;  // staged halo of KTILER_OP_GAUSS_F32 (radius <= 4; 16-B aligned boxes)
struct StageGeo {
  int64_t ry0, xb0, limit;  // limit = roundup16(row bytes) <= pitch
  int nr, stride;
  bool halo;
};
__device__ __forceinline__ int64_t up16(int64_t v) { return (v + 15) & ~(int64_t)15; }
__device__ __forceinline__ StageGeo stage_geo(int op, const DBuf& in, const Tile& t) {
  const int nseg = t.fseg(), rows = t.rows();
  switch (op) {
    case 0: return {t.y0, 3 * t.x0, up16(3 * in.W), rows, 48 * nseg, false};
    case 1: return {t.y0 - 2, t.x0 - 16, up16(in.W), rows + 4, 16 * (nseg + 2), true};
    case 2: return {2 * t.y0, 2 * t.x0, up16(in.W), 2 * rows, 32 * nseg, false};
    case 3: return {t.y0 - 1, t.x0 - 16, up16(in.W), rows + 2, 16 * (nseg + 2), true};
    case 6: return {t.y0 - 1, 4 * (t.x0 - 4), up16(4 * in.W), rows + 2, 4 * (t.fw + 8), true};  // f32, 2 px halo (16-B aligned)
    case 7: return {t.y0 - GAUSS_H, 4 * (t.x0 - GAUSS_H), up16(4 * in.W), rows + 2 * GAUSS_H, 4 * (t.fw + 2 * GAUSS_H), true};
    default: return {t.y0, 4 * t.x0, up16(4 * in.W), rows, 64 * nseg, false};
  }
}

// Shared memory one staged input tile of op needs for an output tile tw x th.
__host__ __device__ inline int stage_bytes(int op, int tw, int th) {
  const int nseg = (tw + 15) / 16;
  switch (op) {
    case 0: return th * 48 * nseg;               // rgb rows, 48 B per 16 px
    case 1: return (th + 4) * 16 * (nseg + 2);   // gray rows y-2..y+2, 16-B halo chunks
    case 2: return 2 * th * 32 * nseg;           // 2 blur rows per output row
    case 3: return (th + 2) * 16 * (nseg + 2);   // down rows y-1..y+1
    case 4: return th * 64 * nseg;               // f32 rows
    case 6: return (th + 2) * 4 * (tw + 8);      // (u, v) rows y-1..y+th, two pixels of halo per side
    case 7: return (th + 2 * GAUSS_H) * 4 * (tw + 2 * GAUSS_H);  // f32 window, GAUSS_H px of halo
  }
  return 0;
}

// Issue the staging of op's input for tile t with one bulk copy per row (TMA), completing
// on mbarrier m.  Called by ONE warp (lane = its lane id); no wait.
__device__ __forceinline__ void stage_issue(int op, const DBuf& in, const Tile& t, uint8_t* sm, uint64_t* m, int lane) {
  const StageGeo g = stage_geo(op, in, t);
  const int64_t lo = g.xb0 > 0 ? g.xb0 : 0;
  const int64_t hi = g.xb0 + g.stride < g.limit ? g.xb0 + g.stride : g.limit;
  const unsigned bytes = (unsigned)(hi - lo);
  if (lane == 0) mbar_arrive_expect(m, bytes * (unsigned)g.nr);
  __syncwarp();
  for (int r = lane; r < g.nr; r += 32) {
    const int64_t y = g.halo ? clampi(g.ry0 + r, 0, in.H - 1) : g.ry0 + r;
    bulk_g2s(sm + r * g.stride + (lo - g.xb0), row_ptr(in, t.z, y) + lo, bytes, m);
  }
}

// Tensor-map TMA (the fast path): ONE cp.async.bulk.tensor.3d per tile, issued by one
// thread.  The map views the input buffer as 4-byte elements [frames][rows][row/4]; the box
// is the whole staged window (stage_geo at full tile size), so out-of-image rows/columns
// of a halo come back zero-filled and are fixed by stage_fix (replicate).  box_bytes is the
// full box (also for ragged edge tiles, whose extra bytes are ignored).
// evict_first: the tile's lines are L2 eviction candidates first (a streamed graph input).
__device__ __forceinline__ void stage_issue_tmap(int op, const CUtensorMap* map, unsigned box_bytes, const DBuf& in,
                                                 const Tile& t, uint8_t* sm, uint64_t* m, bool evict_first = false) {
  const StageGeo g = stage_geo(op, in, t);
  mbar_arrive_expect(m, box_bytes);
  const int x = (int)(g.xb0 >> 2), y = (int)g.ry0, z = (int)(in.ring ? t.z % in.ring : t.z);
  if (evict_first) {
    const uint64_t pol = policy_evict_first();
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, "
        "%3, %4}], [%5], %6;" ::"r"(smem_u32(sm)),
        "l"(map), "r"(x), "r"(y), "r"(z), "r"(smem_u32(m)), "l"(pol)
        : "memory");
  } else {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
            smem_u32(sm)),
        "l"(map), "r"(x), "r"(y), "r"(z), "r"(smem_u32(m))
        : "memory");
  }
}

// After the copies landed (stencils only): replicate-fill the halo outside the image —
// columns < 0 / >= W from pixel 0 / W-1 of the same row, then rows < 0 / >= H as copies of
// the nearest image row — so the staged window holds in[clamp(y)][clamp(x)].  All threads;
// the caller synchronizes afterwards.  Returns quickly for interior tiles.
__device__ __forceinline__ void stage_fix(int op, const DBuf& in, const Tile& t, uint8_t* sm, int nt, int tid,
                                          int bar_id = 4) {
  if (op != 1 && op != 3 && op != 6 && op != 7) return;
  const StageGeo g = stage_geo(op, in, t);
  const int pe = op == 6 ? 8 : (op == 7 ? 4 : 1);                                          // bytes per pixel
  const int ew = op >= 6 ? 4 : 1;                                                          // bytes per element
  const int left = g.xb0 < 0 ? (int)(-g.xb0) : 0;                                          // bytes < 0
  const int rfrom = (int)(ew * in.W - g.xb0) < g.stride ? (int)(ew * in.W - g.xb0) : g.stride;  // bytes >= row end
  const int right = g.stride - rfrom;
  const int top = g.ry0 < 0 ? (int)(-g.ry0) : 0;                                           // rows < 0
  const int bfrom = (int)(in.H - g.ry0) < g.nr ? (int)(in.H - g.ry0) : g.nr;                // rows >= H
  const int per = left + right;
  if (per) {
    for (int i = tid; i < (bfrom - top) * per; i += nt) {
      const int r = top + i / per, k = i % per;
      uint8_t* row = sm + r * g.stride;
      if (k < left) row[k] = row[left + k % pe];                   // pixel 0
      else row[rfrom + (k - left)] = row[rfrom - pe + (k - left) % pe];  // last pixel
    }
  }
  if (top || bfrom < g.nr) {
    if (per) asm volatile("bar.sync %0, %1;" ::"r"(bar_id), "r"(nt) : "memory");  // the nt staging threads only
    const int n16 = g.stride >> 4, nfix = top + (g.nr - bfrom);
    for (int i = tid; i < nfix * n16; i += nt) {
      const int j = i / n16, c = i % n16;
      const int r = j < top ? j : bfrom + (j - top);
      const int src = j < top ? top : bfrom - 1;
      reinterpret_cast<uint4*>(sm + r * g.stride)[c] = reinterpret_cast<const uint4*>(sm + src * g.stride)[c];
    }
  }
}

// Does tile t of a stencil op need stage_fix?  (CTA-uniform)
__device__ __forceinline__ bool needs_fix(int op, const DBuf& in, const Tile& t) {
  if (op != 1 && op != 3 && op != 6 && op != 7) return false;
  const StageGeo g = stage_geo(op, in, t);
  const int64_t rowb = op >= 6 ? 4 * in.W : in.W;
  return g.xb0 < 0 || g.xb0 + g.stride > rowb || g.ry0 < 0 || g.ry0 + g.nr > in.H;
}

__device__ __forceinline__ void store_u8_16(uint8_t* d, int64_t x, int64_t W, uint4 o) {
  if (x + 16 <= W) {
    st16(d, o);
  } else {
    const uint32_t w[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
    for (int k = 0; k < 16; ++k)
      if (x + k < W) d[k] = (uint8_t)(w[k >> 2] >> (8 * (k & 3)));
  }
}

// ---------------------------------------------------------------------------------
// gray: rgb8 -> u8.  Y = (19595R + 38470G + 7471B + 32768) >> 16.  The weights are u16,
// the channels u8: dp2a (two u16 x u8 products + accumulator, lower or upper byte pair of
// the pixel word) takes them straight from the interleaved words, two dp2a per pixel and
// no unpacking.  Pixels 4j..4j+3 live in words (w0, w1, w2) = [R0 G0 B0 R1] [G1 B1 R2 G2]
// [B2 R3 G3 B3]; the weight pairs follow the byte pairs each dp2a sees.  The sum is
// < 2^24, so byte 2 of it is Y.
// ---------------------------------------------------------------------------------
constexpr uint32_t WR = 19595u, WG = 38470u, WB = 7471u;
__device__ __forceinline__ uint32_t pk16(uint32_t lo, uint32_t hi) { return lo | (hi << 16); }
__device__ __forceinline__ void luma4(uint32_t w0, uint32_t w1, uint32_t w2, uint32_t s[4]) {
  s[0] = __dp2a_hi(pk16(WB, 0), w0, __dp2a_lo(pk16(WR, WG), w0, 32768u));   // R0 G0 | B0 (R1)
  s[1] = __dp2a_lo(pk16(WG, WB), w1, __dp2a_hi(pk16(0, WR), w0, 32768u));   // (B0) R1 | G1 B1
  s[2] = __dp2a_lo(pk16(WB, 0), w2, __dp2a_hi(pk16(WR, WG), w1, 32768u));   // R2 G2 | B2 (R3)
  s[3] = __dp2a_hi(pk16(WG, WB), w2, __dp2a_lo(pk16(0, WR), w2, 32768u));   // (B2) R3 | G3 B3
}

__device__ __forceinline__ uint4 gray16(const uint32_t w[12]) {
  uint32_t s[16];
#pragma unroll
  for (int j = 0; j < 4; ++j) luma4(w[3 * j], w[3 * j + 1], w[3 * j + 2], s + 4 * j);
  uint4 o;
  uint32_t* ow = &o.x;
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    uint32_t a = prmt(s[4 * m], s[4 * m + 1], 0x0062);
    uint32_t b = prmt(s[4 * m + 2], s[4 * m + 3], 0x0062);
    ow[m] = prmt(a, b, 0x5410);
  }
  return o;
}

// Items of a tile = (row group g, 16-px column segment s), item it = g * nseg + s, dealt
// round-robin to the CTA's threads.  One loop, so each op's (fully unrolled) item body is
// instantiated once — several copies overflow the instruction cache.  Power-of-two
// segment counts (the B200 geometry) take the shift path for the index split.
template <class F>
__device__ __forceinline__ void for_items(int nseg, int ngrp, int nt, int tid, F&& f) {
  const int total = nseg * ngrp;
  const bool pow2 = (nseg & (nseg - 1)) == 0;
  const int sh = __ffs(nseg) - 1;
  for (int it = tid; it < total; it += nt) {
    const int g = pow2 ? (it >> sh) : it / nseg;
    f(g, it - g * nseg);
  }
}

// Rows per item of the sliding-window stencils: as few row groups as still give every
// thread an item, so the halo rows each item re-reads (4 for blur5, 2 for sobel3) are
// amortised over as many output rows as the CTA's thread count allows.
__device__ __forceinline__ int rows_per_item(int rows, int nseg, int nt) {
  const int ngrp = max(1, nt / nseg);
  return (rows + ngrp - 1) / ngrp;
}

// Output base of a tile (pixel (x0, y0) of frame z) and its "all segments full" flag.
__device__ __forceinline__ uint8_t* tile_out(const DBuf& out, const Tile& t, int elem) {
  return out.p + zoff(out, t.z) + t.y0 * out.pitch + t.x0 * elem;
}

__device__ void gray_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), stride = 48 * t.fseg();
  const bool full = (t.x1 - t.x0) == 16 * nseg;
  uint8_t* const ob = tile_out(out, t, 1);
  const int pitch = (int)out.pitch;
  for_items(nseg, t.rows(), nt, tid, [&](int r, int s) {
    const uint8_t* p = sm + r * stride + 48 * s;
    uint4 a = lds16(p), b = lds16(p + 16), c = lds16(p + 32);
    const uint32_t w[12] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w, c.x, c.y, c.z, c.w};
    uint8_t* d = ob + r * pitch + 16 * s;
    const uint4 o = gray16(w);
    if (full) st16(d, o); else store_u8_16(d, t.x0 + 16 * s, out.W, o);
  });
}

// ---------------------------------------------------------------------------------
// blur5: horizontal [1 4 6 4 1] on packed pairs, then vertical over a 5-row window.
// ---------------------------------------------------------------------------------
// window of 24 bytes [x-4, x+20) of a staged row (p points at the byte of column x)
__device__ __forceinline__ void smem_window(const uint8_t* p, uint32_t t[6]) {
  t[0] = lds4(p - 4);
  uint4 c = lds16(p);
  t[1] = c.x; t[2] = c.y; t[3] = c.z; t[4] = c.w;
  t[5] = lds4(p + 16);
}

// Packed pair (byte at x+j, byte at x+j+1) as u16x2, j in [-4, 18], from the window.
template <int J>
__device__ __forceinline__ uint32_t pair_at(const uint32_t t[6]) {
  constexpr int o = J + 4, q = o >> 2, p = o & 3;
  if constexpr (p == 3) {
    return prmt(t[q], t[q + 1], 0x0403) & 0x00FF00FFu;
  } else {
    return prmt(t[q], 0, 0x4040 + 0x0101 * p + 0x0100);  // [b_p, 0, b_{p+1}, 0]
  }
}

// h[k] = (h[2k], h[2k+1]), h[i] = s[i-2] + 4 s[i-1] + 6 s[i] + 4 s[i+1] + s[i+2] <= 4080.
// Pairs P[i] = (byte x+i-2, byte x+i-1) of the window as u16x2: per window word q,
// L_q = (b0, b1), M_q = (b1, b2), H_q = (b2, b3) are one PRMT each, and the pair that
// straddles words q and q+1 is (H_q.hi, L_{q+1}.lo) — one more PRMT (19 in all).
__device__ __forceinline__ void hblur16(const uint32_t t[6], uint32_t h[8]) {
  uint32_t L[6], M[6], H[6], X[5];
#pragma unroll
  for (int q = 0; q < 6; ++q) {
    if (q >= 1) L[q] = prmt(t[q], 0, 0x4140);
    if (q >= 1 && q <= 4) M[q] = prmt(t[q], 0, 0x4241);
    if (q <= 4) H[q] = prmt(t[q], 0, 0x4342);
  }
#pragma unroll
  for (int q = 0; q < 5; ++q) X[q] = prmt(H[q], L[q + 1], 0x5432);
  // P[i]: window offset o = i + 2 -> word q = o >> 2, byte o & 3 -> H / X / L / M
  uint32_t P[19];
#pragma unroll
  for (int i = 0; i < 19; ++i) {
    const int o = i + 2, q = o >> 2, b = o & 3;
    P[i] = b == 0 ? L[q] : (b == 1 ? M[q] : (b == 2 ? H[q] : X[q]));
  }
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    uint32_t a = P[2 * k] + P[2 * k + 4];
    uint32_t c = P[2 * k + 1] + P[2 * k + 3];
    h[k] = a + 4u * c + 6u * P[2 * k + 2];
  }
}

__device__ __forceinline__ uint4 vblur_pack(const uint32_t* h0, const uint32_t* h1, const uint32_t* h2,
                                           const uint32_t* h3, const uint32_t* h4) {
  uint32_t v[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) v[k] = h0[k] + h4[k] + 0x00800080u + 4u * (h1[k] + h3[k]) + 6u * h2[k];  // <= 65408
  // (v + 128) >> 8 of each lane = byte 1 / byte 3
  return make_uint4(prmt(v[0], v[1], 0x7531), prmt(v[2], v[3], 0x7531), prmt(v[4], v[5], 0x7531),
                    prmt(v[6], v[7], 0x7531));
}

// One item = a 16-px column strip of rpi output rows.  The 5-row window of horizontal
// partials h[] rotates through five register arrays; the row loop is unrolled by 5 so
// every slot index is a compile-time constant (no register moves), whatever rpi is.
__device__ void blur_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), rows = t.rows(), stride = 16 * (t.fseg() + 2);
  const bool full = (t.x1 - t.x0) == 16 * nseg;
  uint8_t* const ob = tile_out(out, t, 1);
  const int pitch = (int)out.pitch;
  const int rpi = rows_per_item(rows, nseg, nt);
  for_items(nseg, (rows + rpi - 1) / rpi, nt, tid, [&](int g, int s) {
    const int ra = g * rpi, n = min(rpi, rows - ra);
    const uint8_t* col = sm + 16 * (s + 1) + ra * stride;  // staged row r holds image row y0 - 2 + r
    uint8_t* d = ob + ra * pitch + 16 * s;
    uint32_t h[5][8];
    uint32_t w[6];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      smem_window(col + i * stride, w);
      hblur16(w, h[i]);
    }
    for (int r0 = 0; r0 < n; r0 += 5) {
#pragma unroll
      for (int k = 0; k < 5; ++k) {
        const int r = r0 + k;
        if (r >= n) break;
        smem_window(col + (r + 4) * stride, w);
        hblur16(w, h[(k + 4) % 5]);
        const uint4 o = vblur_pack(h[k % 5], h[(k + 1) % 5], h[(k + 2) % 5], h[(k + 3) % 5], h[(k + 4) % 5]);
        if (full) st16(d + r * pitch, o); else store_u8_16(d + r * pitch, t.x0 + 16 * s, out.W, o);
      }
    }
  });
}

// ---------------------------------------------------------------------------------
// down2: 2x2 mean, round half up.  16 output pixels from 2 staged rows x 32 bytes.
// ---------------------------------------------------------------------------------
// (sum of the 2x2 block + 2) >> 2 for output pixels 2j, 2j+1 from one word of each input
// row: per word, bytes (0, 2) and (1, 3) as u16x2 lanes (E, O), so E + O holds the two
// horizontal pair sums; two 3-input adds take both rows and the rounding constant.  The
// lanes are < 2^10, so the >> 2 of the packed word moves only garbage into bits 14-15 and
// 30-31: bytes 0 and 2 are the results.
__device__ __forceinline__ uint32_t down2px(uint32_t a, uint32_t b) {
  const uint32_t s = (a & 0x00FF00FFu) + prmt(a, 0, 0x4341) + (b & 0x00FF00FFu) + prmt(b, 0, 0x4341) + 0x00020002u;
  return s >> 2;
}
__device__ __forceinline__ uint32_t down4(uint32_t a0, uint32_t a1, uint32_t b0, uint32_t b1) {
  return prmt(down2px(a0, b0), down2px(a1, b1), 0x6420);
}

__device__ void down_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), stride = 32 * t.fseg();
  const bool full = (t.x1 - t.x0) == 16 * nseg;
  uint8_t* const ob = tile_out(out, t, 1);
  const int pitch = (int)out.pitch;
  for_items(nseg, t.rows(), nt, tid, [&](int r, int s) {
    const uint8_t* p0 = sm + (2 * r) * stride + 32 * s;
    const uint8_t* p1 = p0 + stride;
    uint4 a = lds16(p0), b = lds16(p0 + 16), c = lds16(p1), e = lds16(p1 + 16);
    const uint4 o = make_uint4(down4(a.x, a.y, c.x, c.y), down4(a.z, a.w, c.z, c.w), down4(b.x, b.y, e.x, e.y),
                               down4(b.z, b.w, e.z, e.w));
    uint8_t* d = ob + r * pitch + 16 * s;
    if (full) st16(d, o); else store_u8_16(d, t.x0 + 16 * s, out.W, o);
  });
}

// ---------------------------------------------------------------------------------
// sobel3: u8 -> f32 magnitude, packed 2x16-bit lanes.  For each window word q (window
// bytes 4q..4q+3 = columns x-4+4q .. x-1+4q) keep the even lanes E = (b0, b2) and odd lanes
// O = (b1, b3) of three rows; S = top + 2 mid + bot (<= 1020), D = bot - top + 255.  Then
// for output columns c = x+4q-4 .. x+4q-1 (q = 1..4):
//   even (c, c+2): gx = S(c+1) - S(c-1) = SO_q - (SO_{q-1}.hi, SO_q.lo)
//                  gy = D(c-1) + 2 D(c) + D(c+1) = (DO_{q-1}.hi, DO_q.lo) + 2 DE_q + DO_q
//   odd (c+1, c+3): gx = (SE_q.hi, SE_{q+1}.lo) - SE_q;  gy = DE_q + 2 DO_q + (DE_q.hi, DE_{q+1}.lo)
// with a +1020 bias per lane.  A lane becomes a float exactly as (0x4B000000 | lane) -
// (2^23 + 1020); gx^2 + gy^2 < 2^24 is exact in f32 and sqrt_rn is correctly rounded.
// ---------------------------------------------------------------------------------
struct SobelRow {
  uint32_t e[6], o[6];  // e[1..5] and o[0..4] are used
};
__device__ __forceinline__ void sobel_split(const uint32_t t[6], SobelRow& r) {
#pragma unroll
  for (int q = 0; q < 6; ++q) {
    if (q >= 1) r.e[q] = prmt(t[q], 0, 0x4240);
    if (q <= 4) r.o[q] = prmt(t[q], 0, 0x4341);
  }
}
__device__ __forceinline__ float rsqrt_approx(float x) {
  float y;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// Both lanes of a biased u16x2 word as floats (lane - 1020): (0x4B000000 | lane) is
// 2^23 + lane exactly, one packed f32x2 add removes 2^23 + 1020.
__device__ __forceinline__ float2 lanes_f2(uint32_t w) {
  const float lo = __uint_as_float(prmt(w, 0x4B000000u, 0x7610));
  const float hi = __uint_as_float(prmt(w, 0x4B000000u, 0x7632));
  return __fadd2_rn(make_float2(lo, hi), make_float2(-8389628.0f, -8389628.0f));
}
// Correctly rounded sqrt of two integer-valued floats s in [0, 2*1020^2]: rsqrt.approx,
// then one Newton correction r = g + (s - g^2) * y/2 with g = s*y.  Equal to __fsqrt_rn
// on every integer of that domain — checked exhaustively on the device by
// ktiler_selftest(KTILER_SELFTEST_SQRT) (tests/test_gpu_parity.py).  s = 0 gives 0 (y is
// taken at max(s, 1)).
__device__ __forceinline__ float2 sqrt2_int(float2 s) {
  const float2 y = make_float2(rsqrt_approx(fmaxf(s.x, 1.0f)), rsqrt_approx(fmaxf(s.y, 1.0f)));
  const float2 g = __fmul2_rn(s, y);
  const float2 h = __fmul2_rn(y, make_float2(0.5f, 0.5f));
  const float2 e = __ffma2_rn(make_float2(-g.x, -g.y), g, s);
  return __ffma2_rn(e, h, g);
}
// Magnitudes of the two lanes of biased (gx, gy) words: gx^2 + gy^2 < 2^21 is exact in f32.
__device__ __forceinline__ float2 mag2(uint32_t gx, uint32_t gy) {
  const float2 X = lanes_f2(gx), Y = lanes_f2(gy);
  return sqrt2_int(__ffma2_rn(X, X, __fmul2_rn(Y, Y)));
}

// One item = a 16-px column strip of rpi output rows; the 3-row window rotates through
// three register sets, the row loop unrolled by 3 (static slot indices).
__device__ __forceinline__ void sobel_row(const SobelRow& T, const SobelRow& M, const SobelRow& B, uint8_t* drow,
                                          bool seg_full, int64_t x0, int64_t W) {
  float* dst = reinterpret_cast<float*>(drow);
  // Two halves of 8 columns (window words q = 1, 2 and q = 3, 4), each stored as soon as it
  // is done: at most 8 results and the column sums of words q-1 .. q+1 are live at once
  // (register pressure: 4 sobel CTAs per SM at 128 registers before).
#pragma unroll
  for (int half = 0; half < 2; ++half) {
    uint32_t o[8];  // columns x + 8*half .. x + 8*half + 7
#pragma unroll
    for (int qq = 0; qq < 2; ++qq) {
      const int q = 1 + 2 * half + qq;
      // column smoothing S = top + 2 mid + bot, difference D = bot - top + 255 (per lane)
      const uint32_t SOm = T.o[q - 1] + B.o[q - 1] + 2u * M.o[q - 1];
      const uint32_t SOq = T.o[q] + B.o[q] + 2u * M.o[q];
      const uint32_t SEq = T.e[q] + B.e[q] + 2u * M.e[q];
      const uint32_t SEp = T.e[q + 1] + B.e[q + 1] + 2u * M.e[q + 1];
      const uint32_t DOm = B.o[q - 1] + 0x00FF00FFu - T.o[q - 1];
      const uint32_t DOq = B.o[q] + 0x00FF00FFu - T.o[q];
      const uint32_t DEq = B.e[q] + 0x00FF00FFu - T.e[q];
      const uint32_t DEp = B.e[q + 1] + 0x00FF00FFu - T.e[q + 1];
      const uint32_t gxe = SOq + 0x03FC03FCu - prmt(SOm, SOq, 0x5432);
      const uint32_t gye = prmt(DOm, DOq, 0x5432) + 2u * DEq + DOq;
      const uint32_t gxo = prmt(SEq, SEp, 0x5432) + 0x03FC03FCu - SEq;
      const uint32_t gyo = DEq + 2u * DOq + prmt(DEq, DEp, 0x5432);
      const float2 ev = mag2(gxe, gye);  // columns c, c+2 (c = x + 4q - 4)
      const float2 od = mag2(gxo, gyo);  // columns c+1, c+3
      o[4 * qq + 0] = __float_as_uint(ev.x);
      o[4 * qq + 1] = __float_as_uint(od.x);
      o[4 * qq + 2] = __float_as_uint(ev.y);
      o[4 * qq + 3] = __float_as_uint(od.y);
    }
    if (seg_full) {
      // one 256-bit store per 8 columns: whole 32-B sectors (16-B stores at a 64-B lane
      // stride would write every sector in two halves, doubling the L2 write requests)
      st32(dst + 8 * half, o);
    } else {
#pragma unroll
      for (int k = 0; k < 8; ++k)
        if (x0 + 8 * half + k < W) dst[8 * half + k] = __uint_as_float(o[k]);
    }
  }
}

__device__ void sobel_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), rows = t.rows(), stride = 16 * (t.fseg() + 2);
  const bool full = (t.x1 - t.x0) == 16 * nseg;
  uint8_t* const ob = tile_out(out, t, 4);
  const int pitch = (int)out.pitch;
  const int rpi = rows_per_item(rows, nseg, nt);
  for_items(nseg, (rows + rpi - 1) / rpi, nt, tid, [&](int g, int s) {
    const int ra = g * rpi, n = min(rpi, rows - ra);
    const uint8_t* col = sm + 16 * (s + 1) + ra * stride;  // staged row r holds image row y0 - 1 + r
    uint8_t* drow = ob + ra * pitch + 64 * s;
    const bool seg_full = full || t.x0 + 16 * s + 16 <= out.W;
    const int64_t x0 = t.x0 + 16 * s;
    SobelRow w[3];
    uint32_t tw[6];
    smem_window(col, tw);
    sobel_split(tw, w[0]);
    smem_window(col + stride, tw);
    sobel_split(tw, w[1]);
    for (int r0 = 0; r0 < n; r0 += 3) {
#pragma unroll
      for (int k = 0; k < 3; ++k) {
        const int r = r0 + k;
        if (r >= n) break;
        smem_window(col + (r + 2) * stride, tw);
        sobel_split(tw, w[(k + 2) % 3]);
        sobel_row(w[k % 3], w[(k + 1) % 3], w[(k + 2) % 3], drow + r * pitch, seg_full, x0, out.W);
      }
    }
  });
}

// ---------------------------------------------------------------------------------
// thresh: f32 -> u8 {0,255}, strict >
// ---------------------------------------------------------------------------------
// four f32 pixels -> four bytes {0, 255}: set.gt.u32.f32 gives 0xFFFFFFFF / 0 per pixel
// (IEEE compare: NaN > T is false), byte 0 of each mask packed with three PRMTs
__device__ __forceinline__ uint32_t fset_gt(uint32_t v, float T) {
  uint32_t m;
  asm("set.gt.u32.f32 %0, %1, %2;" : "=r"(m) : "f"(__uint_as_float(v)), "f"(T));
  return m;
}
__device__ __forceinline__ uint32_t gt4(uint4 v, float T) {
  const uint32_t lo = prmt(fset_gt(v.x, T), fset_gt(v.y, T), 0x0040);
  const uint32_t hi = prmt(fset_gt(v.z, T), fset_gt(v.w, T), 0x0040);
  return prmt(lo, hi, 0x5410);
}

__device__ void thresh_compute(const DBuf& out, const Tile& t, const uint8_t* sm, float T, int nt, int tid) {
  const uint64_t pol = policy_evict_first();
  const int nseg = t.nseg(), stride = 64 * t.fseg();
  const bool full = (t.x1 - t.x0) == 16 * nseg;
  uint8_t* const ob = tile_out(out, t, 1);
  const int pitch = (int)out.pitch;
  for_items(nseg, t.rows(), nt, tid, [&](int r, int s) {
    const uint8_t* p = sm + r * stride + 64 * s;
    const uint4 o = make_uint4(gt4(lds16(p), T), gt4(lds16(p + 16), T), gt4(lds16(p + 32), T), gt4(lds16(p + 48), T));
    uint8_t* d = ob + r * pitch + 16 * s;
    if (full) st16_stream(d, o, pol); else store_u8_16(d, t.x0 + 16 * s, out.W, o);
  });
}

// ---------------------------------------------------------------------------------
// jacobi: one Horn-Schunck Jacobi iteration (KTILER_OP_JACOBI, the paper's JI node).  The
// staged window holds (u, v) of rows y0-1 .. y1 with one pixel of halo per side
// (replicate-fixed at image edges); an item = 2 pixels of one row.  Coefficients
// (Ix, Iy, It, -) come straight from global memory (read once, 1:1, 128-bit loads).
// Every operation is an explicitly rounded f32 op in the order of include/ktiler.h, so
// the result is bit-identical to any IEEE evaluation in that order (DESIGN A39).
// ---------------------------------------------------------------------------------
__device__ __forceinline__ float2 jacobi_px(float2 l, float2 r, float2 u, float2 d, float4 c, float a2) {
  const float ub = __fmul_rn(__fadd_rn(__fadd_rn(l.x, r.x), __fadd_rn(u.x, d.x)), 0.25f);
  const float vb = __fmul_rn(__fadd_rn(__fadd_rn(l.y, r.y), __fadd_rn(u.y, d.y)), 0.25f);
  const float num = __fadd_rn(__fadd_rn(__fmul_rn(c.x, ub), __fmul_rn(c.y, vb)), c.z);
  const float den = __fadd_rn(__fadd_rn(a2, __fmul_rn(c.x, c.x)), __fmul_rn(c.y, c.y));
  const float tt = __fdiv_rn(num, den);
  return make_float2(__fsub_rn(ub, __fmul_rn(c.x, tt)), __fsub_rn(vb, __fmul_rn(c.y, tt)));
}

__device__ void jacobi_compute(const DBuf& out, const DBuf& coef, const Tile& t, const uint8_t* sm, float a2, int nt,
                               int tid) {
  const int stride = 4 * (t.fw + 8);           // bytes per staged row (2 px of halo per side)
  const int npair = (int)((t.x1 - t.x0) >> 2);  // pixel pairs per row (x in floats, 4 floats per pair)
  const int rows = t.rows();
  const int64_t px0 = t.x0 >> 1;               // first output pixel
  for (int it = tid; it < npair * rows; it += nt) {
    const int r = it / npair, q = it - r * npair;
    // staged pixel k of a row sits at byte 8 * (k + 2): pixels 2q-2 .. 2q+3 of the centre row
    const uint8_t* cen = sm + (r + 1) * stride + 16 * q;
    const float4 a = *reinterpret_cast<const float4*>(cen);        // pixels 2q-2, 2q-1
    const float4 b = *reinterpret_cast<const float4*>(cen + 16);   // pixels 2q, 2q+1 (unused centre)
    const float4 c = *reinterpret_cast<const float4*>(cen + 32);   // pixels 2q+2, 2q+3
    const float4 up = *reinterpret_cast<const float4*>(cen - stride + 16);  // row above: 2q, 2q+1
    const float4 dn = *reinterpret_cast<const float4*>(cen + stride + 16);  // row below
    const int64_t y = t.y0 + r, x = px0 + 2 * q;
    const float4* cp = reinterpret_cast<const float4*>(coef.p + zoff(coef, t.z) + y * coef.pitch) + x;
    const float4 c0 = __ldcg(cp), c1 = __ldcg(cp + 1);  // every iteration re-reads them: keep in L2
    // pixel 2q: left 2q-1, right 2q+1;  pixel 2q+1: left 2q, right 2q+2
    const float2 o0 = jacobi_px(make_float2(a.z, a.w), make_float2(b.z, b.w), make_float2(up.x, up.y),
                                make_float2(dn.x, dn.y), c0, a2);
    const float2 o1 = jacobi_px(make_float2(b.x, b.y), make_float2(c.x, c.y), make_float2(up.z, up.w),
                                make_float2(dn.z, dn.w), c1, a2);
    float4* dst = reinterpret_cast<float4*>(out.p + zoff(out, t.z) + y * out.pitch) + (x >> 1);
    *dst = make_float4(o0.x, o0.y, o1.x, o1.y);
  }
}

// ---------------------------------------------------------------------------------
// gauss_f32: separable Gaussian on f32 (KTILER_OP_GAUSS_F32, the float variant SURVEY
// §8(c) O-7 describes).  taps[0..2r] are the host's f64-normalised weights rounded to f32
// (r = ceil(3 sigma) <= GAUSS_H).  Horizontal pass over the staged window (rows y0-H ..
// y1+H) into a second shared buffer, a CTA barrier, then the vertical pass; each output is
// an f32 FMA chain in tap order k = -r..r.  Replicate border via stage_fix.
// ---------------------------------------------------------------------------------
// One item = a column strip 4 pixels wide and rows_per_item rows tall.  Each staged row is
// read once (three float4 loads: columns x-4 .. x+7), its horizontal pass kept in a
// (2R+1)-row register window that the unroll-by-(2R+1) row loop rotates with static
// indices, and every output row is one vertical FMA chain over the window — no second
// shared buffer, no CTA barrier.  Tiles cut by the image's right edge (a last strip
// narrower than 4) take the per-pixel path.
template <int R>
__device__ __forceinline__ float4 gauss_hrow(const float* src, const float* wk) {  // src: staged column x (16-B aligned)
  float v[12];  // columns x-4 .. x+7
#pragma unroll
  for (int q = 0; q < 3; ++q) {
    const float4 f = *reinterpret_cast<const float4*>(src - 4 + 4 * q);
    v[4 * q] = f.x; v[4 * q + 1] = f.y; v[4 * q + 2] = f.z; v[4 * q + 3] = f.w;
  }
  float o[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    float a = 0.0f;
#pragma unroll
    for (int k = -R; k <= R; ++k) a = __fmaf_rn(wk[k + R], v[4 + j + k], a);
    o[j] = a;
  }
  return make_float4(o[0], o[1], o[2], o[3]);
}
template <int R>
__device__ __forceinline__ void gauss_compute_r(const DBuf& out, const Tile& t, const uint8_t* sm, const float* taps,
                                                int nt, int tid) {
  static_assert(R >= 1 && R <= GAUSS_H, "radius");
  constexpr int NW = 2 * R + 1;
  const int tw = t.fw, rows = t.rows(), w = (int)(t.x1 - t.x0);
  const int nq = (w + 3) >> 2, sw = tw + 2 * GAUSS_H;
  const float* S = reinterpret_cast<const float*>(sm);  // [rows + 2H][tw + 2H], row r = image row y0 - H + r
  float wk[NW];
#pragma unroll
  for (int k = 0; k < NW; ++k) wk[k] = taps[k];
  float* const ob = reinterpret_cast<float*>(tile_out(out, t, 4));
  const int pitch = (int)(out.pitch >> 2);
  const int ngrp0 = max(1, nt / max(nq, 1));
  const int rpi = (rows + ngrp0 - 1) / ngrp0, ngrp = (rows + rpi - 1) / rpi;
  for (int it = tid; it < nq * ngrp; it += nt) {
    const int g = it / nq, x = 4 * (it - g * nq);
    const int ra = g * rpi, n = min(rpi, rows - ra);
    // output row ra + r needs staged rows ra + r + H - R .. ra + r + H + R
    const float* col = S + (ra + GAUSS_H - R) * sw + GAUSS_H + x;
    float* d = ob + ra * pitch + x;
    if (x + 4 > w) {  // ragged strip: per pixel
      for (int r = 0; r < n; ++r)
        for (int j = 0; x + j < w; ++j) {
          float a = 0.0f;
          for (int i = -R; i <= R; ++i) {
            float h = 0.0f;
            for (int k = -R; k <= R; ++k) h = __fmaf_rn(wk[k + R], col[(r + R + i) * sw + j + k], h);
            a = __fmaf_rn(wk[i + R], h, a);
          }
          d[r * pitch + j] = a;
        }
      continue;
    }
    float4 h[NW];
#pragma unroll
    for (int i = 0; i < NW - 1; ++i) h[i] = gauss_hrow<R>(col + i * sw, wk);
    for (int r0 = 0; r0 < n; r0 += NW) {
#pragma unroll
      for (int k = 0; k < NW; ++k) {
        const int r = r0 + k;
        if (r >= n) break;
        h[(k + NW - 1) % NW] = gauss_hrow<R>(col + (r + NW - 1) * sw, wk);
        float4 a = make_float4(0.0f, 0.0f, 0.0f, 0.0f);
#pragma unroll
        for (int i = 0; i < NW; ++i) {
          const float4 v = h[(k + i) % NW];
          a.x = __fmaf_rn(wk[i], v.x, a.x);
          a.y = __fmaf_rn(wk[i], v.y, a.y);
          a.z = __fmaf_rn(wk[i], v.z, a.z);
          a.w = __fmaf_rn(wk[i], v.w, a.w);
        }
        *reinterpret_cast<float4*>(d + r * pitch) = a;
      }
    }
  }
}
__device__ void gauss_compute(const DBuf& out, const Tile& t, const uint8_t* sm, const float* taps, int r, int nt,
                              int tid) {
  switch (r) {
    case 1: gauss_compute_r<1>(out, t, sm, taps, nt, tid); break;
    case 2: gauss_compute_r<2>(out, t, sm, taps, nt, tid); break;
    case 3: gauss_compute_r<3>(out, t, sm, taps, nt, tid); break;
    default: gauss_compute_r<4>(out, t, sm, taps, nt, tid); break;
  }
}

// Compute op's output tile from its staged input (after the staging is complete).
__device__ __forceinline__ void compute_tile(int op, const DBuf& out, const Tile& t, const uint8_t* sm, float T,
                                             int nt, int tid, const DBuf* aux = nullptr, const float* taps = nullptr,
                                             int radius = 0) {
  switch (op) {
    case 0: gray_compute(out, t, sm, nt, tid); break;
    case 1: blur_compute(out, t, sm, nt, tid); break;
    case 2: down_compute(out, t, sm, nt, tid); break;
    case 3: sobel_compute(out, t, sm, nt, tid); break;
    case 4: thresh_compute(out, t, sm, T, nt, tid); break;
    case 6: jacobi_compute(out, *aux, t, sm, T, nt, tid); break;  // T = a2 (alpha^2)
    case 7: gauss_compute(out, t, sm, taps, radius, nt, tid); break;
  }
}

// One whole block (stream / graph modes): stage (TMA), wait, fix edges, compute.
// m: an mbarrier in shared memory initialised with count 1 (phase 0 unused before).
__device__ __forceinline__ void run_tile(int op, bool scalar, const DBuf& in, const DBuf& out, const Tile& t, float T,
                                         int nt, int tid, uint8_t* sm, uint64_t* m) {
  if (scalar) {
    scalar_tile(op, in, out, t, T, nt, tid);
    return;
  }
  if (tid < 32) stage_issue(op, in, t, sm, m, tid);
  mbar_wait(m, 0);
  stage_fix(op, in, t, sm, nt, tid);
  __syncthreads();
  compute_tile(op, out, t, sm, T, nt, tid);
}

}  // namespace ktd
