/*
 * oracle/ktiler_oracle.c — KTILER result oracle (plain C99, single thread).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load, link or call this file.  The
 * product path (paper_conf_date_maghazeh0ep19_b200/) never touches it and shares
 * no code, header, table or constant with it.
 *
 * KTILER (Maghazeh et al., DATE 2019) computes exactly the untiled result, only
 * faster: "instead of having each kernel process the entire input in one
 * invocation, we subdivide the input into fragments" (Abstract).  So
 * the result oracle is the plain definition of each kernel, run over whole images
 * in topological order (the paper's "normal execution mode").  The
 * five kernels are the north star's (BASELINE.json north_star); the paper names
 * only "converted to a grayscale image" and "scaled down" — every
 * reading of an unstated detail is SURVEY §8(c) A1–A7 and is listed in
 * DESIGN.md §2.  Compiled -O2 -fno-fast-math -ffp-contract=off.
 *
 * Each kernel is written once, as a per-pixel function whose memory accesses go
 * through the rd8/rdf/wr8/wrf accessors.  Three drivers use it:
 *   - ko_run_rect: computes every output pixel of one rectangle (a whole image
 *     = the untiled kernel; one block's output rect = the block-granular executor
 *     O-9 the tests use to replay any schedule on poisoned buffers);
 *   - the same with tracing on (O-10): each written byte remembers its writer
 *     block, each read looks the writer up -> exact RAW block dependencies
 *     ("B depends on B' iff a thread in B reads a memory address previously
 *     written by a thread in B'") and the 128-B memory lines each
 *     block touches — a CPU re-enactment of the SASSI trace
 *     (PAPER.md:219–223);
 *   - ko_pipeline: the whole untiled graph (O-6), used for the CPU baseline.
 *
 * Pins (tests/test_oracle_pins.py): library routines (Pillow convert('L'),
 * cv2.resize INTER_AREA / PIL reduce(2), cv2.GaussianBlur(5x5, BORDER_REPLICATE),
 * cv2.Sobel), closed forms, and the hand-worked 4x4 / 8x8 fixtures under
 * tests/golden/.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { KO_GRAY = 0, KO_BLUR5 = 1, KO_DOWN2 = 2, KO_SOBEL3 = 3, KO_THRESH = 4 };

/* A dense image buffer: [F][H][W][elem] bytes.  base = simulated byte address
 * of element 0 (used only to compute 128-B memory lines when tracing). */
typedef struct {
  void* data;
  int64_t W, H, F, elem;
  int64_t base;
  int32_t id;
  int32_t pad;
} ko_buf;

/* ------------------------------------------------------------------------- */
/* tracing state (O-10)                                                      */
/* ------------------------------------------------------------------------- */
#define KO_MAXBUF 16
static int g_trace = 0;
static int64_t g_cur = -1;                    /* current block id              */
static int32_t* g_writer[KO_MAXBUF];          /* per byte: writer block or -1  */
static int64_t g_wbytes[KO_MAXBUF];
static int64_t* g_dep = 0;                    /* pairs (consumer, producer)    */
static int64_t g_ndep = 0, g_capdep = 0;
static int64_t* g_line = 0;                   /* pairs (block, line*2+is_write)*/
static int64_t g_nline = 0, g_capline = 0;
static int64_t g_last_dep_w = -2, g_last_line = -1;

static void push2(int64_t** arr, int64_t* n, int64_t* cap, int64_t a, int64_t b) {
  if (*n == *cap) {
    *cap = *cap ? *cap * 2 : 4096;
    *arr = (int64_t*)realloc(*arr, (size_t)(*cap) * 2 * sizeof(int64_t));
  }
  (*arr)[2 * *n] = a;
  (*arr)[2 * *n + 1] = b;
  (*n)++;
}

static void trace_access(const ko_buf* b, int64_t off, int64_t nbytes, int is_write) {
  for (int64_t k = 0; k < nbytes; ++k) {
    int64_t line = (((b->base + off + k) >> 7) << 1) | (is_write ? 1 : 0); /* 128-B lines */
    if (line != g_last_line) {
      push2(&g_line, &g_nline, &g_capline, g_cur, line);
      g_last_line = line;
    }
    int32_t* w = g_writer[b->id];
    if (is_write) {
      w[off + k] = (int32_t)g_cur;
    } else {
      int64_t p = w[off + k];
      if (p >= 0 && p != g_last_dep_w) {
        push2(&g_dep, &g_ndep, &g_capdep, g_cur, p);
        g_last_dep_w = p;
      }
    }
  }
}

static inline int64_t clampi(int64_t v, int64_t lo, int64_t hi) { return v < lo ? lo : (v > hi ? hi : v); }

static inline uint8_t rd8(const ko_buf* b, int64_t z, int64_t y, int64_t x, int64_t c) {
  int64_t off = ((z * b->H + y) * b->W + x) * b->elem + c;
  if (g_trace) trace_access(b, off, 1, 0);
  return ((const uint8_t*)b->data)[off];
}
static inline float rdf(const ko_buf* b, int64_t z, int64_t y, int64_t x) {
  int64_t off = ((z * b->H + y) * b->W + x) * 4;
  if (g_trace) trace_access(b, off, 4, 0);
  float v;
  memcpy(&v, (const uint8_t*)b->data + off, 4);
  return v;
}
static inline void wr8(ko_buf* b, int64_t z, int64_t y, int64_t x, uint8_t v) {
  int64_t off = ((z * b->H + y) * b->W + x) * b->elem;
  if (g_trace) trace_access(b, off, 1, 1);
  ((uint8_t*)b->data)[off] = v;
}
static inline void wrf(ko_buf* b, int64_t z, int64_t y, int64_t x, float v) {
  int64_t off = ((z * b->H + y) * b->W + x) * 4;
  if (g_trace) trace_access(b, off, 4, 1);
  memcpy((uint8_t*)b->data + off, &v, 4);
}

/* ------------------------------------------------------------------------- */
/* the five kernels, one output pixel each                                    */
/* ------------------------------------------------------------------------- */

/* O-1 gray (kernel "A"; weights/rounding = SURVEY A2):
 * Y = (19595 R + 38470 G + 7471 B + 32768) >> 16, BT.601 luma in 16-bit fixed
 * point with round-half-up (== Pillow convert('L')). */
static void px_gray(const ko_buf* in, ko_buf* out, int64_t z, int64_t y, int64_t x) {
  uint32_t R = rd8(in, z, y, x, 0), G = rd8(in, z, y, x, 1), B = rd8(in, z, y, x, 2);
  wr8(out, z, y, x, (uint8_t)((19595u * R + 38470u * G + 7471u * B + 32768u) >> 16));
}

/* O-2 blur5 (north star "separable Gaussian blur"): 5x5 binomial
 * w = [1,4,6,4,1], out = (sum_i sum_j w_i w_j g[clamp(y+i-2)][clamp(x+j-2)] + 128) >> 8,
 * replicate border.  Written as the plain 2-D sum (the definition); the
 * separable order is an exact integer identity. */
static const int32_t W5[5] = {1, 4, 6, 4, 1};
static void px_blur5(const ko_buf* in, ko_buf* out, int64_t z, int64_t y, int64_t x) {
  int32_t s = 0;
  for (int i = 0; i < 5; ++i)
    for (int j = 0; j < 5; ++j)
      s += W5[i] * W5[j] * (int32_t)rd8(in, z, clampi(y + i - 2, 0, in->H - 1), clampi(x + j - 2, 0, in->W - 1), 0);
  wr8(out, z, y, x, (uint8_t)((s + 128) >> 8));
}

/* O-3 down2 (kernel "B": "scaled down to an image of 128x128", PAPER.md:37;
 * filter = SURVEY A3): 2x2 box mean, round half up. */
static void px_down2(const ko_buf* in, ko_buf* out, int64_t z, int64_t y, int64_t x) {
  uint32_t a = rd8(in, z, 2 * y, 2 * x, 0), b = rd8(in, z, 2 * y, 2 * x + 1, 0);
  uint32_t c = rd8(in, z, 2 * y + 1, 2 * x, 0), d = rd8(in, z, 2 * y + 1, 2 * x + 1, 0);
  wr8(out, z, y, x, (uint8_t)((a + b + c + d + 2) >> 2));
}

/* O-4 sobel3: 3x3 Sobel with replicate border,
 * mag = sqrtf((float)(gx^2 + gy^2)); the integer sum is < 2^24 so its float
 * conversion is exact and IEEE sqrt is correctly rounded. */
static void px_sobel3(const ko_buf* in, ko_buf* out, int64_t z, int64_t y, int64_t x) {
  int64_t ym = clampi(y - 1, 0, in->H - 1), yp = clampi(y + 1, 0, in->H - 1);
  int64_t xm = clampi(x - 1, 0, in->W - 1), xp = clampi(x + 1, 0, in->W - 1);
  int32_t p00 = rd8(in, z, ym, xm, 0), p01 = rd8(in, z, ym, x, 0), p02 = rd8(in, z, ym, xp, 0);
  int32_t p10 = rd8(in, z, y, xm, 0), p12 = rd8(in, z, y, xp, 0);
  int32_t p20 = rd8(in, z, yp, xm, 0), p21 = rd8(in, z, yp, x, 0), p22 = rd8(in, z, yp, xp, 0);
  int32_t gx = (p02 + 2 * p12 + p22) - (p00 + 2 * p10 + p20);
  int32_t gy = (p20 + 2 * p21 + p22) - (p00 + 2 * p01 + p02);
  wrf(out, z, y, x, sqrtf((float)(gx * gx + gy * gy)));
}

/* O-5 thresh: strict >, {0, 255}. */
static void px_thresh(const ko_buf* in, ko_buf* out, int64_t z, int64_t y, int64_t x, float T) {
  wr8(out, z, y, x, rdf(in, z, y, x) > T ? 255 : 0);
}

/* ------------------------------------------------------------------------- */
/* drivers                                                                    */
/* ------------------------------------------------------------------------- */

/* Compute every output pixel of op in [x0,x1) x [y0,y1) of frame z.  The rect
 * is clipped to the output buffer.  Returns 0, or -1 for a bad op. */
int ko_run_rect(int op, const ko_buf* in, ko_buf* out, int64_t z, int64_t x0, int64_t y0, int64_t x1,
                int64_t y1, float T) {
  if (x1 > out->W) x1 = out->W;
  if (y1 > out->H) y1 = out->H;
  if (x0 < 0) x0 = 0;
  if (y0 < 0) y0 = 0;
  for (int64_t y = y0; y < y1; ++y)
    for (int64_t x = x0; x < x1; ++x) {
      switch (op) {
        case KO_GRAY: px_gray(in, out, z, y, x); break;
        case KO_BLUR5: px_blur5(in, out, z, y, x); break;
        case KO_DOWN2: px_down2(in, out, z, y, x); break;
        case KO_SOBEL3: px_sobel3(in, out, z, y, x); break;
        case KO_THRESH: px_thresh(in, out, z, y, x, T); break;
        default: return -1;
      }
    }
  return 0;
}

/* O-6: the untiled 5-kernel graph, kernel by kernel over whole images, frame by
 * frame.  rgb [F][H][W][3] -> gray, blur [F][H][W] -> down [F][H/2][W/2] ->
 * sob (f32) -> mask [F][H/2][W/2].  Any intermediate pointer may not be NULL. */
int ko_pipeline(const uint8_t* rgb, int64_t W, int64_t H, int64_t F, float T, uint8_t* gray, uint8_t* blur,
                uint8_t* down, float* sob, uint8_t* mask) {
  if ((W & 1) || (H & 1)) return -1;
  ko_buf b_rgb = {(void*)rgb, W, H, F, 3, 0, 0, 0};
  ko_buf b_gray = {gray, W, H, F, 1, 0, 1, 0};
  ko_buf b_blur = {blur, W, H, F, 1, 0, 2, 0};
  ko_buf b_down = {down, W / 2, H / 2, F, 1, 0, 3, 0};
  ko_buf b_sob = {sob, W / 2, H / 2, F, 4, 0, 4, 0};
  ko_buf b_mask = {mask, W / 2, H / 2, F, 1, 0, 5, 0};
  for (int64_t z = 0; z < F; ++z) {
    ko_run_rect(KO_GRAY, &b_rgb, &b_gray, z, 0, 0, W, H, T);
    ko_run_rect(KO_BLUR5, &b_gray, &b_blur, z, 0, 0, W, H, T);
    ko_run_rect(KO_DOWN2, &b_blur, &b_down, z, 0, 0, W / 2, H / 2, T);
    ko_run_rect(KO_SOBEL3, &b_down, &b_sob, z, 0, 0, W / 2, H / 2, T);
    ko_run_rect(KO_THRESH, &b_sob, &b_mask, z, 0, 0, W / 2, H / 2, T);
  }
  return 0;
}

/* ---- tracing API (O-10) ------------------------------------------------- */
int ko_trace_begin(int32_t nbufs, const int64_t* buf_bytes) {
  if (nbufs > KO_MAXBUF) return -1;
  for (int i = 0; i < KO_MAXBUF; ++i) {
    free(g_writer[i]);
    g_writer[i] = 0;
    g_wbytes[i] = 0;
  }
  for (int i = 0; i < nbufs; ++i) {
    g_wbytes[i] = buf_bytes[i];
    g_writer[i] = (int32_t*)malloc((size_t)(buf_bytes[i] > 0 ? buf_bytes[i] : 1) * sizeof(int32_t));
    for (int64_t k = 0; k < buf_bytes[i]; ++k) g_writer[i][k] = -1;
  }
  g_ndep = g_nline = 0;
  g_trace = 1;
  return 0;
}
void ko_trace_set_block(int64_t gid) {
  g_cur = gid;
  g_last_dep_w = -2;
  g_last_line = -1;
}
void ko_trace_stop(void) { g_trace = 0; }
int64_t ko_trace_ndeps(void) { return g_ndep; }
int64_t ko_trace_nlines(void) { return g_nline; }
void ko_trace_get(int64_t* deps, int64_t* lines) {
  if (deps) memcpy(deps, g_dep, (size_t)g_ndep * 2 * sizeof(int64_t));
  if (lines) memcpy(lines, g_line, (size_t)g_nline * 2 * sizeof(int64_t));
}
