// A USER kernel for the KTILER_OP_CUSTOM tests: an asymmetric 2 x 5 box
// filter on u8, replicate border,
//     out[y][x] = (sum_{dy = 0..1} sum_{dx = -2..2} in[min(y+dy, H-1)][clamp(x+dx)] + 5) / 10
// whose footprint libktiler does not know: the tests declare the node with a naive
// footprint, let ktiler_discover_footprint find the real one (rows y..y+1, columns x-2..x+2
// of each output pixel), fit the affine map and re-plan.  Launched through the
// ktiler_launch_fn callback below.  Test infrastructure, not product code.
#include <cuda_runtime.h>

#include <cstdint>

struct BoxUser {  // the callback's `user` (host memory, owned by the test)
  const uint8_t* in;
  uint8_t* out;
  int64_t W, H, pitch_in, pitch_out, fs_in, fs_out;
  int32_t tw, th;
};

constexpr int MAXR = 16;
struct BoxLaunch {
  BoxUser u;
  int32_t n;
  int32_t r[MAXR][6];
  int64_t pre[MAXR + 1];
};

__global__ void asym_box_kernel(const __grid_constant__ BoxLaunch L) {
  int k = 0;
  const int64_t b = blockIdx.x;
  while (k + 1 < L.n && b >= L.pre[k + 1]) ++k;
  const int32_t* r = L.r[k];
  const int64_t lin = b - L.pre[k], w = r[3] - r[0], h = r[4] - r[1];
  const int64_t bx = r[0] + lin % w, by = r[1] + (lin / w) % h, bz = r[2] + lin / (w * h);
  const BoxUser& u = L.u;
  const int64_t x0 = bx * u.tw, y0 = by * u.th;
  for (int i = threadIdx.x; i < u.tw * u.th; i += blockDim.x) {
    const int64_t x = x0 + i % u.tw, y = y0 + i / u.tw;
    if (x >= u.W || y >= u.H) continue;
    int s = 5;
    for (int dy = 0; dy <= 1; ++dy) {
      const int64_t yy = y + dy < u.H ? y + dy : u.H - 1;
      const uint8_t* row = u.in + bz * u.fs_in + yy * u.pitch_in;
      for (int dx = -2; dx <= 2; ++dx) {
        int64_t xx = x + dx;
        xx = xx < 0 ? 0 : (xx >= u.W ? u.W - 1 : xx);
        s += row[xx];
      }
    }
    u.out[bz * u.fs_out + y * u.pitch_out + x] = (uint8_t)(s / 10);
  }
}

extern "C" void asym_box_launch(void* user, const int32_t* rects, int32_t n, void* stream) {
  for (int32_t c = 0; c < n; c += MAXR) {
    BoxLaunch L;
    L.u = *static_cast<const BoxUser*>(user);
    L.n = n - c < MAXR ? n - c : MAXR;
    L.pre[0] = 0;
    for (int i = 0; i < L.n; ++i) {
      for (int j = 0; j < 6; ++j) L.r[i][j] = rects[6 * (c + i) + j];
      L.pre[i + 1] = L.pre[i] + (int64_t)(L.r[i][3] - L.r[i][0]) * (L.r[i][4] - L.r[i][1]) * (L.r[i][5] - L.r[i][2]);
    }
    if (L.pre[L.n] > 0) asym_box_kernel<<<(unsigned)L.pre[L.n], 256, 0, (cudaStream_t)stream>>>(L);
  }
}
