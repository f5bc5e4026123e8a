// L2 (LTS) throughput microbenchmark — the secondary ceiling of SURVEY §8(d): every byte
// of the tiled schedule (hits and misses alike) passes through the L2 slices, so their
// throughput, not HBM, bounds a schedule whose intermediates stay resident.
//
// Modes, each over a buffer of `mb` MiB touched once beforehand (resident when mb << L2):
//   read   : every thread streams 16-B ld.global.cg loads over the buffer, XOR-reduced
//   write  : 16-B st.global over the buffer
//   copy   : read half A, write half B (the op kernels' pattern)
//   write_evict_last / write_evict_unchanged : the write with an L2 createpolicy hint
//   write256 / read256 : 32 B per thread per instruction (STG.E.256 / LDG.E.256)
// Grid = 148 x 8 CTAs x 256 threads, grid-stride, 20 passes per launch (resident sizes);
// CUDA events around `iters` launches;
// prints one JSON line per mode with bytes / time.  Diagnostic tool, not product code.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/l2bw tools/l2bw.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>

__global__ void rd(const uint4* __restrict__ p, size_t n, unsigned* sink, int reps) {
  uint32_t acc = 0;
  for (int k = 0; k < reps; ++k)
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v;
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p + i));
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678u) *sink = acc;
}
__global__ void wr(uint4* __restrict__ p, size_t n, unsigned salt, int reps) {
  for (int k = 0; k < reps; ++k)
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = make_uint4(salt + k, (unsigned)i, salt, (unsigned)i);
}
// resident writes with an L2 eviction-priority hint (createpolicy): evict_last / evict_unchanged
__global__ void wr_hint(uint4* __restrict__ p, size_t n, unsigned salt, int reps, int hint) {
  uint64_t pol;
  if (hint == 0) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  else asm volatile("createpolicy.fractional.L2::evict_unchanged.b64 %0, 1.0;" : "=l"(pol));
  for (int k = 0; k < reps; ++k)
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
      asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p + i), "r"(salt + k), "r"((unsigned)i),
                   "r"(salt), "r"((unsigned)i), "l"(pol)
                   : "memory");
}
// resident writes, 32 B per thread per instruction (st.global.v8.b32 = STG.E.256)
__global__ void wr256(uint4* __restrict__ p, size_t n, unsigned salt, int reps) {
  for (int k = 0; k < reps; ++k)
    for (size_t i = 2 * (blockIdx.x * (size_t)blockDim.x + threadIdx.x); i + 1 < n; i += 2 * (size_t)gridDim.x * blockDim.x)
      asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p + i), "r"(salt + k), "r"((unsigned)i),
                   "r"(salt), "r"((unsigned)i), "r"(salt), "r"(salt), "r"(salt), "r"(salt)
                   : "memory");
}
// resident reads, 32 B per thread per instruction (ld.global.cg.v8.b32)
__global__ void rd256(const uint4* __restrict__ p, size_t n, unsigned* sink, int reps) {
  uint32_t acc = 0;
  for (int k = 0; k < reps; ++k)
    for (size_t i = 2 * (blockIdx.x * (size_t)blockDim.x + threadIdx.x); i + 1 < n; i += 2 * (size_t)gridDim.x * blockDim.x) {
      uint32_t v[8];
      asm volatile("ld.global.cg.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                   : "l"(p + i));
      acc ^= v[0] ^ v[1] ^ v[2] ^ v[3] ^ v[4] ^ v[5] ^ v[6] ^ v[7];
    }
  if (acc == 0x12345678u) *sink = acc;
}

// resident writes, each 128-B line dropped right after it is written (discard.global.L2:
// invalidate without write-back).  Lanes 8g..8g+7 write one line; lane 8g drops it after
// the warp barrier.  Tests whether the write ceiling is the L2 write path or the eager
// write-back of dirty lines to HBM.
__global__ void wr_disc(uint4* __restrict__ p, size_t n, unsigned salt, int reps) {
  const int lane = threadIdx.x & 31;
  for (int k = 0; k < reps; ++k)
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
      p[i] = make_uint4(salt + k, (unsigned)i, salt, (unsigned)i);
      __syncwarp();
      if ((lane & 7) == 0) asm volatile("discard.global.L2 [%0], 128;" ::"l"(p + i) : "memory");
    }
}
// resident writes by the bulk-copy engine: cp.async.bulk.global.shared::cta (UBLKCP S2G),
// CHUNK bytes per copy from one shared buffer, one issuing thread per CTA
template <int CHUNK>
__global__ void wr_bulk(uint4* __restrict__ p, size_t n, int reps, int disc) {
  __shared__ __align__(128) uint8_t sm[CHUNK];
  for (int i = threadIdx.x; i < CHUNK / 4; i += blockDim.x) reinterpret_cast<unsigned*>(sm)[i] = i * 2654435761u;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  const size_t nch = n * 16 / CHUNK;
  const unsigned s = (unsigned)__cvta_generic_to_shared(sm);
  if (threadIdx.x == 0) {
    for (int k = 0; k < reps; ++k)
      for (size_t c = blockIdx.x; c < nch; c += gridDim.x) {
        uint8_t* g = reinterpret_cast<uint8_t*>(p) + c * CHUNK;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(g), "r"(s), "r"(CHUNK) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 8;" ::: "memory");
      }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  if (disc) {  // drop what this CTA wrote (after its bulk writes completed)
    __syncthreads();
    for (int k = 0; k < 1; ++k)
      for (size_t c = blockIdx.x; c < nch; c += gridDim.x)
        for (int l = threadIdx.x; l < CHUNK / 128; l += blockDim.x)
          asm volatile("discard.global.L2 [%0], 128;" ::"l"(reinterpret_cast<uint8_t*>(p) + c * CHUNK + 128 * l) : "memory");
  }
}

__global__ void cp(const uint4* __restrict__ a, uint4* __restrict__ b, size_t n, int reps) {
  for (int k = 0; k < reps; ++k)
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v;
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(a + i));
    b[i] = v;
  }
}

static const char* NAMES[] = {"read", "write", "copy", "write_evict_last", "write_evict_unchanged", "write256",
                              "read256", "write_discard", "bulk_s2g_4k", "bulk_s2g_16k", "bulk_s2g_16k_discard"};
constexpr int NMODES = 11;

// usage: l2bw [mode ...]  (names above; default all) ; env L2BW_MB = "32,4096" sizes
int main(int argc, char** argv) {
  const int iters = getenv("L2BW_ITERS") ? atoi(getenv("L2BW_ITERS")) : 50;
  size_t sizes_mb[16] = {4, 8, 16, 32, 64, 96, 4096};
  int nsz = 7;
  if (const char* e = getenv("L2BW_MB")) {
    nsz = 0;
    for (const char* q = e; *q && nsz < 16;) {
      sizes_mb[nsz++] = strtoull(q, (char**)&q, 10);
      if (*q == ',') ++q;
    }
  }
  bool want[NMODES];
  for (int m = 0; m < NMODES; ++m) want[m] = argc <= 1;
  for (int a = 1; a < argc; ++a)
    for (int m = 0; m < NMODES; ++m)
      if (!strcmp(argv[a], NAMES[m])) want[m] = true;
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  uint4* buf;
  unsigned* sink;
  cudaMalloc(&buf, (size_t)4096 << 20);
  cudaMalloc(&sink, 4);
  cudaMemset(buf, 1, (size_t)4096 << 20);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int grid = nsm * 8, block = 256;
  for (int si = 0; si < nsz; ++si) {
    const size_t mb = sizes_mb[si];
    const size_t n = (mb << 20) / 16;
    const int it = mb > 1024 ? 5 : iters;
    const int reps = mb > 1024 ? 1 : 20;  // passes per launch (no launch gaps in the resident cases)
    for (int mode = 0; mode < NMODES; ++mode) {
      if (!want[mode]) continue;
      auto run = [&]() {
        if (mode == 0) rd<<<grid, block>>>(buf, n, sink, reps);
        else if (mode == 1) wr<<<grid, block>>>(buf, n, 7u, reps);
        else if (mode == 2) cp<<<grid, block>>>(buf, buf + n / 2, n / 2, reps);
        else if (mode < 5) wr_hint<<<grid, block>>>(buf, n, 7u, reps, mode - 3);
        else if (mode == 5) wr256<<<grid, block>>>(buf, n, 7u, reps);
        else if (mode == 6) rd256<<<grid, block>>>(buf, n, sink, reps);
        else if (mode == 7) wr_disc<<<grid, block>>>(buf, n, 7u, reps);
        else if (mode == 8) wr_bulk<4096><<<nsm * 4, 128>>>(buf, n, reps, 0);
        else if (mode == 9) wr_bulk<16384><<<nsm * 4, 128>>>(buf, n, reps, 0);
        else wr_bulk<16384><<<nsm * 4, 128>>>(buf, n, reps, 1);
      };
      run();
      run();
      cudaEventRecord(e0);
      for (int i = 0; i < it; ++i) run();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      const double bytes = (double)(mb << 20) * it * reps;  // copy: n/2 read + n/2 written = mb
      printf("{\"tool\": \"l2bw\", \"mode\": \"%s\", \"mb\": %zu, \"GBps\": %.1f, \"us_per_pass\": %.2f}\n",
             NAMES[mode], mb, bytes / (ms * 1e-3) / 1e9, ms * 1e3 / (it * reps));
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    fprintf(stderr, "%s\n", cudaGetErrorString(e));
    return 1;
  }
  return 0;
}
