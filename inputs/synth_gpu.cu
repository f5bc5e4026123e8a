// Device twin of inputs/synth.py (seeded synthetic RGB8 inputs).
// Holds none of KTILER's arithmetic; it exists only so multi-GB benchmark inputs
// can be generated in HBM instead of uploaded.  Same counter-based generator as
// the numpy version; tests/test_gpu_parity.py::test_gpu_generator_matches_numpy checks them byte for byte.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

constexpr uint64_t K_SEED = 0xD1B54A32D192ED03ull;
constexpr uint64_t K_NOISE = 0x632BE59BD9B4E019ull;

struct Rects {
  int32_t r[64][7];  // x0, y0, x1, y1, R, G, B
};

// rows [y0, y0+rows) of global image rows, frames [f0, f0+F) of a global batch.
__global__ void gen_uniform(uint8_t* dst, int64_t pitch, int64_t frame_stride, int64_t W, int64_t H,
                            int64_t y0, int64_t rows, int64_t f0, uint64_t seed) {
  int64_t f = blockIdx.z;
  uint64_t off = seed * K_SEED;
  for (int64_t y = blockIdx.y; y < rows; y += gridDim.y)
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < W * 3; b += (int64_t)gridDim.x * blockDim.x) {
    uint64_t i = (uint64_t)((((f0 + f) * H + (y0 + y)) * W) * 3 + b);
    dst[f * frame_stride + y * pitch + b] = (uint8_t)(splitmix64(i + off) & 0xFF);
  }
}

__global__ void gen_scene(uint8_t* dst, int64_t pitch, int64_t W, int64_t H, int64_t y0, int64_t rows, uint64_t s,
                          Rects rc) {
  for (int64_t y = blockIdx.y; y < rows; y += gridDim.y) {
  int64_t gy = y0 + y;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < W; x += (int64_t)gridDim.x * blockDim.x) {
    int32_t c[3] = {(int32_t)(x * 255 / W), (int32_t)(gy * 255 / H), 128};
    for (int k = 0; k < 64; ++k) {
      if (x >= rc.r[k][0] && gy >= rc.r[k][1] && x < rc.r[k][2] && gy < rc.r[k][3]) {
        c[0] = rc.r[k][4]; c[1] = rc.r[k][5]; c[2] = rc.r[k][6];
      }
    }
    for (int ch = 0; ch < 3; ++ch) {
      uint64_t i = (uint64_t)((gy * W + x) * 3 + ch);
      int32_t n = (int32_t)(splitmix64(i + s * K_NOISE) & 15) - 8;
      int32_t v = c[ch] + n;
      v = v < 0 ? 0 : (v > 255 ? 255 : v);
      dst[y * pitch + x * 3 + ch] = (uint8_t)v;
    }
  }
  }
}

}  // namespace

extern "C" {

// Returns 0 on success, else the cudaError_t value.
int ktin_gen_uniform(void* dst, int64_t pitch, int64_t frame_stride, int64_t W, int64_t H, int64_t y0,
                     int64_t rows, int64_t f0, int64_t F, uint64_t seed, void* stream) {
  if (rows <= 0 || F <= 0 || W <= 0) return 0;
  dim3 grid((unsigned)((W * 3 + 255) / 256 < 64 ? (W * 3 + 255) / 256 : 64), (unsigned)(rows < 65535 ? rows : 65535), (unsigned)F);
  gen_uniform<<<grid, 256, 0, (cudaStream_t)stream>>>((uint8_t*)dst, pitch, frame_stride, W, H, y0, rows, f0, seed);
  return (int)cudaGetLastError();
}

// One frame; rects = 64*7 int32 (host) from inputs.synth.scene_rects(s, W, H).
int ktin_gen_scene(void* dst, int64_t pitch, int64_t W, int64_t H, int64_t y0, int64_t rows, uint64_t s,
                   const int32_t* rects, void* stream) {
  if (rows <= 0 || W <= 0) return 0;
  Rects rc;
  for (int k = 0; k < 64; ++k)
    for (int j = 0; j < 7; ++j) rc.r[k][j] = rects[k * 7 + j];
  dim3 grid((unsigned)((W + 255) / 256 < 32 ? (W + 255) / 256 : 32), (unsigned)(rows < 65535 ? rows : 65535), 1);
  gen_scene<<<grid, 256, 0, (cudaStream_t)stream>>>((uint8_t*)dst, pitch, W, H, y0, rows, s, rc);
  return (int)cudaGetLastError();
}

}  // extern "C"
