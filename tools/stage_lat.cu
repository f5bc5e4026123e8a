// Staging latency of one 32 KB tile per CTA from an L2-resident buffer, by mechanism:
//   bulk1   one cp.async.bulk (UBLKCP) of 32 KB            (what a 1-box TMA copy does)
//   bulk64  64 cp.async.bulk of 512 B (one per tile row)
//   ldg     128 threads x 16 LDG.128 into registers, then STS (no async proxy)
//   ldgsts  128 threads x 16 cp.async.cg 16 B (LDGSTS), one commit/wait
//   tma_WxR one cp.async.bulk.tensor.2d box of W bytes x R rows (W*R = 32 KB) from a pitched
//           buffer (pitch P bytes; P == W: the box is contiguous) — the op kernels' staging
// Each CTA records (start, staged, end) with %globaltimer; the tool prints per mechanism and
// grid (1 CTA/SM, 8 CTAs/SM, many waves) the mean / p10 / p50 / p90 staging latency and the
// kernel's effective bandwidth (events).  DESIGN.md §6.10 (why L2-fed CTAs are no faster).
// Diagnostic tool, not product code.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
//   -o build/stage_lat tools/stage_lat.cu
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

constexpr int TILE = 32768;
constexpr int NT = 128;

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void __launch_bounds__(NT) stage(const uint8_t* __restrict__ src, size_t nbytes, unsigned long long* rec,
                                            unsigned* sink) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) unsigned long long mbar;
  __shared__ unsigned long long t0;
  const int tid = threadIdx.x;
  if (tid == 0) {
    t0 = gtimer();
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar)));
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  const size_t off = ((size_t)blockIdx.x * TILE) % nbytes;
  const uint8_t* g = src + off;
  if (MODE == 0 || MODE == 1) {
    if (tid == 0) {
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&mbar)), "r"(TILE) : "memory");
      const int n = MODE == 0 ? 1 : 64, sz = TILE / n;
      for (int i = 0; i < n; ++i)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_u32(sm + i * sz)),
            "l"(g + (size_t)i * sz), "r"(sz), "r"(smem_u32(&mbar))
            : "memory");
    }
    unsigned ok = 0;
    while (!ok)
      asm volatile(
          "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
          : "=r"(ok)
          : "r"(smem_u32(&mbar))
          : "memory");
  } else if (MODE == 2) {
    uint4 v[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) v[k] = __ldcg(reinterpret_cast<const uint4*>(g) + k * NT + tid);
#pragma unroll
    for (int k = 0; k < 16; ++k) reinterpret_cast<uint4*>(sm)[k * NT + tid] = v[k];
    __syncthreads();
  } else {
#pragma unroll
    for (int k = 0; k < 16; ++k)
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(sm + 16 * (k * NT + tid))),
                   "l"(g + 16 * (k * NT + tid))
                   : "memory");
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
    __syncthreads();
  }
  const unsigned long long ts = gtimer();
  // consume the tile (so nothing is optimised away)
  unsigned acc = 0;
  for (int k = tid; k < TILE / 16; k += NT) acc ^= reinterpret_cast<const uint4*>(sm)[k].x;
  if (acc == 0x12345678u) atomicAdd(sink, 1u);
  __syncthreads();
  if (tid == 0) {
    rec[3 * blockIdx.x] = t0;
    rec[3 * blockIdx.x + 1] = ts;
    rec[3 * blockIdx.x + 2] = gtimer();
  }
}

__global__ void __launch_bounds__(NT) stage_tma(const __grid_constant__ CUtensorMap map, int bw, int bh, int gx, int gy,
                                                unsigned long long* rec, unsigned* sink) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) unsigned long long mbar;
  __shared__ unsigned long long t0;
  const int tid = threadIdx.x;
  if (tid == 0) {
    t0 = gtimer();
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar)));
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  if (tid == 0) {
    const int b = blockIdx.x % (gx * gy);
    const int x = (b % gx) * (bw / 4), y = (b / gx) * bh;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&mbar)), "r"(TILE) : "memory");
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            smem_u32(sm)),
        "l"(&map), "r"(x), "r"(y), "r"(smem_u32(&mbar))
        : "memory");
  }
  unsigned ok = 0;
  while (!ok)
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                 : "=r"(ok)
                 : "r"(smem_u32(&mbar))
                 : "memory");
  const unsigned long long ts = gtimer();
  unsigned acc = 0;
  for (int k = tid; k < TILE / 16; k += NT) acc ^= reinterpret_cast<const uint4*>(sm)[k].x;
  if (acc == 0x12345678u) atomicAdd(sink, 1u);
  __syncthreads();
  if (tid == 0) {
    rec[3 * blockIdx.x] = t0;
    rec[3 * blockIdx.x + 1] = ts;
    rec[3 * blockIdx.x + 2] = gtimer();
  }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static void report(const char* name, int grid, int nsm, const unsigned long long* rec, float ms) {
  std::vector<unsigned long long> h(3 * (size_t)grid);
  cudaMemcpy(h.data(), rec, h.size() * 8, cudaMemcpyDeviceToHost);
  std::vector<double> st(grid);
  double mean = 0, mt = 0;
  for (int i = 0; i < grid; ++i) {
    st[i] = (double)(h[3 * i + 1] - h[3 * i]) / 1e3;
    mean += st[i];
    mt += (double)(h[3 * i + 2] - h[3 * i]) / 1e3;
  }
  mean /= grid;
  mt /= grid;
  std::sort(st.begin(), st.end());
  printf("{\"tool\": \"stage_lat\", \"mode\": \"%s\", \"grid\": %d, \"ctas_per_sm\": %.0f, \"stage_us_mean\": %.3f, "
         "\"p10\": %.3f, \"p50\": %.3f, \"p90\": %.3f, \"cta_us_mean\": %.3f, \"GBps\": %.1f}\n",
         name, grid, (double)grid / nsm, mean, st[grid / 10], st[grid / 2], st[grid * 9 / 10], mt,
         (double)grid * TILE / (ms * 1e-3) / 1e9);
}

typedef void (*kfn)(const uint8_t*, size_t, unsigned long long*, unsigned*);

int main() {
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const size_t nbytes = 32ull << 20;  // L2-resident source
  uint8_t* src;
  unsigned* sink;
  cudaMalloc(&src, nbytes);
  cudaMemset(src, 1, nbytes);
  cudaMalloc(&sink, 4);
  const int grids[3] = {nsm, 8 * nsm, 64 * nsm};
  unsigned long long* rec;
  cudaMalloc(&rec, sizeof(unsigned long long) * 3 * grids[2]);
  const kfn fns[4] = {stage<0>, stage<1>, stage<2>, stage<3>};
  const char* names[4] = {"bulk1", "bulk64", "ldg", "ldgsts"};
  for (int m = 0; m < 4; ++m) cudaFuncSetAttribute(fns[m], cudaFuncAttributeMaxDynamicSharedMemorySize, TILE);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int gi = 0; gi < 3; ++gi) {
    const int grid = grids[gi];
    for (int m = 0; m < 4; ++m) {
      for (int w = 0; w < 3; ++w) fns[m]<<<grid, NT, TILE>>>(src, nbytes, rec, sink);  // warm L2
      cudaEventRecord(e0);
      fns[m]<<<grid, NT, TILE>>>(src, nbytes, rec, sink);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      report(names[m], grid, nsm, rec, ms);
    }
  }
  // tensor-map boxes: (box bytes per row, rows, buffer pitch, L2 promotion)
  void* ef = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ef, cudaEnableDefault, &q);
  EncodeFn enc = (EncodeFn)ef;
  cudaFuncSetAttribute(stage_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, TILE);
  const int cases[][4] = {{512, 64, 7680, 3}, {1024, 32, 7680, 3}, {256, 128, 7680, 3}, {512, 64, 512, 3},
                          {1024, 32, 1024, 3}, {512, 64, 7680, 0}, {512, 64, 7680, 1}};
  for (const auto& c : cases) {
    const int bw = c[0], bh = c[1], pitch = c[2];
    const int rows = (int)(nbytes / pitch);
    CUtensorMap map;
    cuuint64_t dims[2] = {(cuuint64_t)(pitch / 4), (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)pitch};
    cuuint32_t box[2] = {(cuuint32_t)(bw / 4), (cuuint32_t)bh}, es[2] = {1, 1};
    const CUtensorMapL2promotion pr[4] = {CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_64B,
                                          CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B};
    if (!enc || enc(&map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, src, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_NONE, pr[c[3]], CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      printf("{\"tool\": \"stage_lat\", \"error\": \"encode %dx%d pitch %d\"}\n", bw, bh, pitch);
      continue;
    }
    const int gx = pitch / bw, gy = rows / bh;
    char name[64];
    snprintf(name, sizeof(name), "tma_%dx%d_pitch%d_prom%d", bw, bh, pitch, c[3] == 3 ? 256 : (c[3] == 0 ? 0 : 64));
    for (int gi = 0; gi < 3; ++gi) {
      const int grid = grids[gi];
      for (int w = 0; w < 3; ++w) stage_tma<<<grid, NT, TILE>>>(map, bw, bh, gx, gy, rec, sink);
      cudaEventRecord(e0);
      stage_tma<<<grid, NT, TILE>>>(map, bw, bh, gx, gy, rec, sink);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      report(name, grid, nsm, rec, ms);
    }
  }
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    fprintf(stderr, "CUDA error %s\n", cudaGetErrorString(e));
    return 1;
  }
  return 0;
}
