// sm_100a tile bodies of the five built-in kernels (SURVEY §8(a) a7–a11).
//
// Every body computes ONE block's output rect [x0,x1) x [y0,y1) of frame z with nt
// threads (thread tid); the rect is exactly the block's declared WRITE footprint, so the
// planner's dependency analysis and the kernels can never disagree.
//
// Vector variant (B200 geometry) = two phases, so the persistent executor can overlap
// the memory of one tile with the arithmetic of another:
//   stage_tile    the block's input footprint (+ halo, replicate-clamped at image edges)
//                 into shared memory with cp.async.cg: every 16-B chunk of the tile in
//                 flight at once, L2-only (so data other CTAs produced in the same
//                 persistent launch is never read from a stale L1); no wait;
//   compute_tile  one work item = 16 output pixels of one row (gray, down2, thresh) or a
//                 16-pixel column strip of R rows with a sliding row window in registers
//                 (blur5, sobel3); packed 2x16-bit SIMD arithmetic in 32-bit registers,
//                 byte permutes (PRMT) to unpack/pack, dp4a for the luma dot product,
//                 128-bit stores.
// Scalar variant: the paper's Fig. 1 geometry, one thread per pixel.
// Cache policy: the graph input (rgb) is read once -> L2 evict_first; the graph output
// (mask) is never re-read -> L2 evict_first stores; intermediates keep the default policy
// so they stay resident for their consumer sub-kernel (the point of KTILER).
// Border: replicate (clamp-to-edge) at image edges only.
#pragma once

#include <cstdint>

namespace ktd {

struct DBuf {
  uint8_t* p;
  int64_t W, H, pitch, fstride;
};

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
__device__ __forceinline__ void discard_line(const void* p) {
  asm volatile("discard.global.L2 [%0], 128;" ::"l"(p) : "memory");
}
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async16_hint(void* smem, const void* gmem, uint64_t pol) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "l"(pol) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

__device__ __forceinline__ int64_t clampi(int64_t v, int64_t lo, int64_t hi) { return v < lo ? lo : (v > hi ? hi : v); }
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t s) { return __byte_perm(a, b, s); }
__device__ __forceinline__ const uint8_t* row_ptr(const DBuf& b, int64_t z, int64_t y) {
  return b.p + z * b.fstride + y * b.pitch;
}
__device__ __forceinline__ uint4 lds16(const uint8_t* p) { return *reinterpret_cast<const uint4*>(p); }
__device__ __forceinline__ uint32_t lds4(const uint8_t* p) { return *reinterpret_cast<const uint32_t*>(p); }

struct Tile {
  int64_t z, x0, y0, x1, y1;  // output rect [x0,x1) x [y0,y1) of frame z
  __device__ int nseg() const { return (int)((x1 - x0 + 15) >> 4); }
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
constexpr int BLUR_R = 8;
constexpr int SOBEL_R = 2;

// Shared memory one staged input tile of op needs for an output tile tw x th.
__host__ __device__ inline int stage_bytes(int op, int tw, int th) {
  const int nseg = (tw + 15) / 16;
  switch (op) {
    case 0: return th * 48 * nseg;               // rgb rows, 48 B per 16 px
    case 1: return (th + 4) * 16 * (nseg + 2);   // gray rows y-2..y+2, 16-B halo chunks
    case 2: return 2 * th * 32 * nseg;           // 2 blur rows per output row
    case 3: return (th + 2) * 16 * (nseg + 2);   // down rows y-1..y+1
    case 4: return th * 64 * nseg;               // f32 rows
  }
  return 0;
}

// Row-contiguous staging: nr rows starting at image row ry0 (step 1), byte span
// [xb, xb + cpr*16) per row, only chunks that start inside the row's data (< limit); the
// chunk end never passes the pitch (pitch >= roundup16(width*elem)).
__device__ __forceinline__ void stage_rows(const DBuf& in, int64_t z, int64_t ry0, int nr, int64_t xb, int cpr,
                                           int64_t limit, uint8_t* sm, int nt, int tid, bool stream, uint64_t pol) {
  const int total = nr * cpr;
  for (int i = tid; i < total; i += nt) {
    const int r = i / cpr, c = i - r * cpr;
    const int64_t off = xb + 16 * c;
    if (off < limit) {
      const uint8_t* src = row_ptr(in, z, ry0 + r) + off;
      uint8_t* dst = sm + r * (16 * cpr) + 16 * c;
      // (cp.async with an L2::cache_hint operand mis-encodes its descriptor register in
      // this toolchain -> illegal instruction on sm_100a; the read-once input goes plain)
      (void)stream;
      (void)pol;
      cp_async16(dst, src);
    }
  }
}

// Halo staging of a u8 tile: rows [ya, ya+nr) (clamped to [0,H)) and byte columns
// [xs, xs + 16*nc) (clamped, replicate), row stride 16*nc.  Interior chunks move with
// cp.async.cg; chunks crossing an image edge are gathered byte by byte.
__device__ __forceinline__ void stage_halo(const DBuf& in, int64_t z, int64_t ya, int nr, int64_t xs, int nc,
                                           uint8_t* sm, int nt, int tid) {
  const int total = nr * nc;
  for (int i = tid; i < total; i += nt) {
    const int r = i / nc, c = i - r * nc;
    const uint8_t* row = row_ptr(in, z, clampi(ya + r, 0, in.H - 1));
    const int64_t x = xs + 16 * c;
    uint8_t* d = sm + r * (16 * nc) + 16 * c;
    if (x >= 0 && x + 16 <= in.W) {
      cp_async16(d, row + x);
    } else {
      uint32_t w[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint32_t v = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j) v |= (uint32_t)ld1(row + clampi(x + 4 * q + j, 0, in.W - 1)) << (8 * j);
        w[q] = v;
      }
      *reinterpret_cast<uint4*>(d) = make_uint4(w[0], w[1], w[2], w[3]);
    }
  }
}

// Issue the staging of op's input for tile t (no wait; the caller commits / waits).
__device__ __forceinline__ void stage_tile(int op, const DBuf& in, const Tile& t, uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), rows = t.rows();
  switch (op) {
    case 0: stage_rows(in, t.z, t.y0, rows, 3 * t.x0, 3 * nseg, 3 * in.W, sm, nt, tid, true, policy_evict_first()); break;
    case 1: stage_halo(in, t.z, t.y0 - 2, rows + 4, t.x0 - 16, nseg + 2, sm, nt, tid); break;
    case 2: stage_rows(in, t.z, 2 * t.y0, 2 * rows, 2 * t.x0, 2 * nseg, in.W, sm, nt, tid, false, 0); break;
    case 3: stage_halo(in, t.z, t.y0 - 1, rows + 2, t.x0 - 16, nseg + 2, sm, nt, tid); break;
    case 4: stage_rows(in, t.z, t.y0, rows, 4 * t.x0, 4 * nseg, 4 * in.W, sm, nt, tid, false, 0); break;
  }
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
// gray: rgb8 -> u8.  Y = (19595R + 38470G + 7471B + 32768) >> 16 computed as
// 256*dp4a(px, [76,150,29,0]) + dp4a(px, [139,70,47,0]) + 32768, whose byte 2 is Y
// (19595 = 76*256+139, 38470 = 150*256+70, 7471 = 29*256+47; the sum is < 2^24).
// ---------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t luma_sum(uint32_t px) {
  uint32_t hi = __dp4a(px, 0x001D964Cu, 0u);
  uint32_t lo = __dp4a(px, 0x002F468Bu, 32768u);
  return hi * 256u + lo;
}

__device__ __forceinline__ uint4 gray16(const uint32_t w[12]) {
  uint32_t s[16];
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    const int b = 3 * k, q = b >> 2, sh = b & 3;
    // bytes 3k..3k+2 into bytes 0..2 (byte 3 has weight 0 in both dot products)
    uint32_t px = sh == 0 ? w[q] : (sh == 1 ? (w[q] >> 8) : prmt(w[q], w[q + 1], 0x3210 + 0x1111 * sh));
    s[k] = luma_sum(px);
  }
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

__device__ void gray_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), items = nseg * t.rows(), stride = 48 * nseg;
  for (int it = tid; it < items; it += nt) {
    const int r = it / nseg, s = it - r * nseg;
    const uint8_t* p = sm + r * stride + 48 * s;
    uint4 a = lds16(p), b = lds16(p + 16), c = lds16(p + 32);
    const uint32_t w[12] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w, c.x, c.y, c.z, c.w};
    const int64_t x = t.x0 + 16 * s;
    store_u8_16(const_cast<uint8_t*>(row_ptr(out, t.z, t.y0 + r)) + x, x, out.W, gray16(w));
  }
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
__device__ __forceinline__ void hblur16(const uint32_t t[6], uint32_t h[8]) {
  uint32_t P[19];
  P[0] = pair_at<-2>(t); P[1] = pair_at<-1>(t); P[2] = pair_at<0>(t); P[3] = pair_at<1>(t);
  P[4] = pair_at<2>(t); P[5] = pair_at<3>(t); P[6] = pair_at<4>(t); P[7] = pair_at<5>(t);
  P[8] = pair_at<6>(t); P[9] = pair_at<7>(t); P[10] = pair_at<8>(t); P[11] = pair_at<9>(t);
  P[12] = pair_at<10>(t); P[13] = pair_at<11>(t); P[14] = pair_at<12>(t); P[15] = pair_at<13>(t);
  P[16] = pair_at<14>(t); P[17] = pair_at<15>(t); P[18] = pair_at<16>(t);
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    uint32_t a = P[2 * k] + P[2 * k + 4];
    uint32_t b = P[2 * k + 1] + P[2 * k + 3];
    h[k] = a + 4u * b + 6u * P[2 * k + 2];
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

template <int R>
__device__ void blur_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), rows = t.rows(), stride = 16 * (nseg + 2);
  const int ngrp = (rows + R - 1) / R, items = nseg * ngrp;
  for (int it = tid; it < items; it += nt) {
    const int g = it / nseg, s = it - g * nseg;
    const int ra = g * R, rb = min(ra + R, rows);
    const uint8_t* col = sm + 16 * (s + 1);  // staged row r holds image row y0 - 2 + r
    const int64_t x = t.x0 + 16 * s;
    uint32_t h[5][8];
    uint32_t w[6];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      smem_window(col + (ra + i) * stride, w);
      hblur16(w, h[i]);
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (ra + r >= rb) break;
      smem_window(col + (ra + r + 4) * stride, w);
      hblur16(w, h[(r + 4) % 5]);
      uint4 o = vblur_pack(h[r % 5], h[(r + 1) % 5], h[(r + 2) % 5], h[(r + 3) % 5], h[(r + 4) % 5]);
      store_u8_16(const_cast<uint8_t*>(row_ptr(out, t.z, t.y0 + ra + r)) + x, x, out.W, o);
    }
  }
}

// ---------------------------------------------------------------------------------
// down2: 2x2 mean, round half up.  16 output pixels from 2 staged rows x 32 bytes.
// ---------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t hsum2(uint32_t w) {  // (b0+b1, b2+b3) as u16x2
  return (w & 0x00FF00FFu) + ((w >> 8) & 0x00FF00FFu);
}
__device__ __forceinline__ uint32_t down4(uint32_t a0, uint32_t a1, uint32_t b0, uint32_t b1) {
  uint32_t lo = ((hsum2(a0) + hsum2(b0) + 0x00020002u) >> 2) & 0x00FF00FFu;
  uint32_t hi = ((hsum2(a1) + hsum2(b1) + 0x00020002u) >> 2) & 0x00FF00FFu;
  return prmt(lo, hi, 0x6420);
}

__device__ void down_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), items = nseg * t.rows(), stride = 32 * nseg;
  for (int it = tid; it < items; it += nt) {
    const int r = it / nseg, s = it - r * nseg;
    const uint8_t* p0 = sm + (2 * r) * stride + 32 * s;
    const uint8_t* p1 = p0 + stride;
    uint4 a = lds16(p0), b = lds16(p0 + 16), c = lds16(p1), e = lds16(p1 + 16);
    const uint4 o = make_uint4(down4(a.x, a.y, c.x, c.y), down4(a.z, a.w, c.z, c.w), down4(b.x, b.y, e.x, e.y),
                               down4(b.z, b.w, e.z, e.w));
    const int64_t x = t.x0 + 16 * s;
    store_u8_16(const_cast<uint8_t*>(row_ptr(out, t.z, t.y0 + r)) + x, x, out.W, o);
  }
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
  uint32_t e[6], o[6];
};
__device__ __forceinline__ void sobel_split(const uint32_t t[6], SobelRow& r) {
#pragma unroll
  for (int q = 0; q < 6; ++q) {
    r.e[q] = prmt(t[q], 0, 0x4240);
    r.o[q] = prmt(t[q], 0, 0x4341);
  }
}
__device__ __forceinline__ float lane_f(uint32_t w, bool hi) {
  const float f = __uint_as_float(prmt(w, 0x4B000000u, hi ? 0x7632 : 0x7610));
  return f - 8389628.0f;  // 2^23 + 1020
}
__device__ __forceinline__ float mag(float gx, float gy) { return __fsqrt_rn(__fmaf_rn(gx, gx, __fmul_rn(gy, gy))); }

template <int R>
__device__ void sobel_compute(const DBuf& out, const Tile& t, const uint8_t* sm, int nt, int tid) {
  const int nseg = t.nseg(), rows = t.rows(), stride = 16 * (nseg + 2);
  const int ngrp = (rows + R - 1) / R, items = nseg * ngrp;
  for (int it = tid; it < items; it += nt) {
    const int g = it / nseg, s = it - g * nseg;
    const int ra = g * R, rb = min(ra + R, rows);
    const uint8_t* col = sm + 16 * (s + 1);  // staged row r holds image row y0 - 1 + r
    const int64_t x = t.x0 + 16 * s;
    SobelRow w[3];
    uint32_t tw[6];
    smem_window(col + ra * stride, tw);
    sobel_split(tw, w[0]);
    smem_window(col + (ra + 1) * stride, tw);
    sobel_split(tw, w[1]);
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (ra + r >= rb) break;
      smem_window(col + (ra + r + 2) * stride, tw);
      sobel_split(tw, w[(r + 2) % 3]);
      const SobelRow& T = w[r % 3];
      const SobelRow& M = w[(r + 1) % 3];
      const SobelRow& B = w[(r + 2) % 3];
      uint32_t SE[6], SO[6], DE[6], DO[6];
#pragma unroll
      for (int q = 0; q < 6; ++q) {
        SE[q] = T.e[q] + 2u * M.e[q] + B.e[q];
        SO[q] = T.o[q] + 2u * M.o[q] + B.o[q];
        DE[q] = B.e[q] + 0x00FF00FFu - T.e[q];
        DO[q] = B.o[q] + 0x00FF00FFu - T.o[q];
      }
      float* dst = reinterpret_cast<float*>(const_cast<uint8_t*>(row_ptr(out, t.z, t.y0 + ra + r))) + x;
      float m[16];
#pragma unroll
      for (int q = 1; q <= 4; ++q) {
        const uint32_t gxe = SO[q] + 0x03FC03FCu - prmt(SO[q - 1], SO[q], 0x5432);
        const uint32_t gye = prmt(DO[q - 1], DO[q], 0x5432) + 2u * DE[q] + DO[q];
        const uint32_t gxo = prmt(SE[q], SE[q + 1], 0x5432) + 0x03FC03FCu - SE[q];
        const uint32_t gyo = DE[q] + 2u * DO[q] + prmt(DE[q], DE[q + 1], 0x5432);
        const int b = 4 * (q - 1);
        m[b + 0] = mag(lane_f(gxe, false), lane_f(gye, false));
        m[b + 1] = mag(lane_f(gxo, false), lane_f(gyo, false));
        m[b + 2] = mag(lane_f(gxe, true), lane_f(gye, true));
        m[b + 3] = mag(lane_f(gxo, true), lane_f(gyo, true));
      }
      if (x + 16 <= out.W) {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          st16(dst + 4 * q, make_uint4(__float_as_uint(m[4 * q]), __float_as_uint(m[4 * q + 1]),
                                       __float_as_uint(m[4 * q + 2]), __float_as_uint(m[4 * q + 3])));
      } else {
#pragma unroll
        for (int k = 0; k < 16; ++k)
          if (x + k < out.W) dst[k] = m[k];
      }
    }
  }
}

// ---------------------------------------------------------------------------------
// thresh: f32 -> u8 {0,255}, strict >
// ---------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t gt4(uint4 v, float T) {
  uint32_t a = __uint_as_float(v.x) > T ? 0xFFu : 0u, b = __uint_as_float(v.y) > T ? 0xFFu : 0u;
  uint32_t c = __uint_as_float(v.z) > T ? 0xFFu : 0u, d = __uint_as_float(v.w) > T ? 0xFFu : 0u;
  return a | (b << 8) | (c << 16) | (d << 24);
}

__device__ void thresh_compute(const DBuf& out, const Tile& t, const uint8_t* sm, float T, int nt, int tid) {
  const uint64_t pol = policy_evict_first();
  const int nseg = t.nseg(), items = nseg * t.rows(), stride = 64 * nseg;
  for (int it = tid; it < items; it += nt) {
    const int r = it / nseg, s = it - r * nseg;
    const uint8_t* p = sm + r * stride + 64 * s;
    const uint4 o = make_uint4(gt4(lds16(p), T), gt4(lds16(p + 16), T), gt4(lds16(p + 32), T), gt4(lds16(p + 48), T));
    const int64_t x = t.x0 + 16 * s;
    uint8_t* d = const_cast<uint8_t*>(row_ptr(out, t.z, t.y0 + r)) + x;
    if (x + 16 <= out.W) st16_stream(d, o, pol); else store_u8_16(d, x, out.W, o);
  }
}

// Compute op's output tile from its staged input (after the staging is complete).
__device__ __forceinline__ void compute_tile(int op, const DBuf& out, const Tile& t, const uint8_t* sm, float T,
                                             int nt, int tid) {
  switch (op) {
    case 0: gray_compute(out, t, sm, nt, tid); break;
    case 1: blur_compute<BLUR_R>(out, t, sm, nt, tid); break;
    case 2: down_compute(out, t, sm, nt, tid); break;
    case 3: sobel_compute<SOBEL_R>(out, t, sm, nt, tid); break;
    case 4: thresh_compute(out, t, sm, T, nt, tid); break;
  }
}

// One whole block (stream / graph modes): stage, wait, compute.
__device__ __forceinline__ void run_tile(int op, bool scalar, const DBuf& in, const DBuf& out, const Tile& t, float T,
                                         int nt, int tid, uint8_t* sm) {
  if (scalar) {
    scalar_tile(op, in, out, t, T, nt, tid);
    return;
  }
  stage_tile(op, in, t, sm, nt, tid);
  cp_async_commit();
  cp_async_wait<0>();
  __syncthreads();
  compute_tile(op, out, t, sm, T, nt, tid);
}

}  // namespace ktd
