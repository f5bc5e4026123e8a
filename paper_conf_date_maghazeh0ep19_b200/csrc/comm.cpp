// Strip halo exchange (BASELINE configs[4]: "a single giant image shards
// into horizontal strips whose halo rows move over NVLink via NCCL send/recv").
//
// Rank r of n owns full-resolution rows [o0, o1) of the image and holds its *extended*
// strip [e0, e1) = its rows plus the halo rows above and below (the chain's reach, 4 rgb
// rows; strips.py).  Before the tiled schedule runs, the one exchange step of the path
// fills the halo rows from the neighbours:
//   receive rows [e0, o0) from rank r-1 (its last owned rows) and rows [o1, e1) from r+1;
//   send my first / last min(h, o1 - o0) owned rows to r-1 / r+1.
// Two backends behind one handle:
//   NCCL      one rank per process and GPU: ncclSend / ncclRecv of the contiguous row
//             blocks inside one ncclGroupStart/End (NVLink / NVSwitch peer transport);
//             libnccl is resolved at run time with dlopen — the copy torch has already
//             loaded when there is one (one NCCL per process), else libnccl.so.2.
//   LOOPBACK  n emulated ranks on ONE device (tests and the 1-GPU evidence): every rank's
//             strip is registered, and the exchange is the same row-block moves as one
//             cudaMemcpy2DAsync per halo.
// Both are stream-ordered and capturable, so ktiler_plan_attach_halo puts the exchange
// into the same CUDA graph as the schedule (ktiler_execute = exchange + tiled graph).
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>  // types only; every function is resolved with dlsym

#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "kt_internal.h"

using kt::fail;

namespace {

struct NcclApi {
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
  bool ok = false;
  std::string why;
};

const NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);  // the process's NCCL (torch's)
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      api.why = "libnccl.so.2 not found";
      return;
    }
    auto sym = [&](const char* n) { return dlsym(h, n); };
    api.GetUniqueId = (decltype(api.GetUniqueId))sym("ncclGetUniqueId");
    api.CommInitRank = (decltype(api.CommInitRank))sym("ncclCommInitRank");
    api.CommDestroy = (decltype(api.CommDestroy))sym("ncclCommDestroy");
    api.Send = (decltype(api.Send))sym("ncclSend");
    api.Recv = (decltype(api.Recv))sym("ncclRecv");
    api.GroupStart = (decltype(api.GroupStart))sym("ncclGroupStart");
    api.GroupEnd = (decltype(api.GroupEnd))sym("ncclGroupEnd");
    api.GetErrorString = (decltype(api.GetErrorString))sym("ncclGetErrorString");
    api.CommGetAsyncError = (decltype(api.CommGetAsyncError))sym("ncclCommGetAsyncError");
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.Send && api.Recv && api.GroupStart &&
             api.GroupEnd && api.GetErrorString;
    if (!api.ok) api.why = "libnccl.so.2 lacks a needed symbol";
  });
  return api;
}

ktiler_status nccl_fail(ncclResult_t r, const char* what) {
  const NcclApi& a = nccl();
  return fail(KTILER_E_CUDA, std::string(what) + ": " + (a.GetErrorString ? a.GetErrorString(r) : "NCCL error"));
}

}  // namespace

struct ktiler_comm_s {
  int kind = KTILER_COMM_LOOPBACK;
  int nranks = 1;
  int rank = 0;  // NCCL: this process's rank
  ncclComm_t nc = nullptr;
  std::vector<ktiler_strip> strips;  // per rank (LOOPBACK: all; NCCL: this rank's)
  std::vector<uint8_t> have;
  ~ktiler_comm_s() {
    if (nc && nccl().CommDestroy) nccl().CommDestroy(nc);
  }
};

namespace kt {

// Row-block geometry of one rank's exchange (see the file comment).
struct HaloRows {
  int64_t recv_top, recv_bot, send_up, send_down;
};
static HaloRows halo_rows_of(const ktiler_strip& s, int rank, int nranks, int32_t h) {
  HaloRows r;
  const int64_t own = s.o1 - s.o0;
  r.recv_top = rank > 0 ? s.o0 - s.e0 : 0;
  r.recv_bot = rank < nranks - 1 ? s.e1 - s.o1 : 0;
  r.send_up = rank > 0 ? std::min<int64_t>(h, own) : 0;
  r.send_down = rank < nranks - 1 ? std::min<int64_t>(h, own) : 0;
  return r;
}
static uint8_t* row_at(const ktiler_strip& s, int64_t y) {  // global row y of the extended strip
  return (uint8_t*)s.base + (y - s.e0) * s.pitch_bytes;
}

// The exchange of `rank` on `st` (also called from exec.cu inside graph capture).
ktiler_status halo_exchange(ktiler_comm_s* c, int32_t rank, int32_t h, void* stream) {
  cudaStream_t st = (cudaStream_t)stream;
  if (!c || rank < 0 || rank >= c->nranks || h < 0) return fail(KTILER_E_INVALID, "bad comm, rank or halo rows");
  if (c->kind == KTILER_COMM_NCCL && rank != c->rank) return fail(KTILER_E_INVALID, "NCCL comm: exchange this rank's strip");
  const int slot = c->kind == KTILER_COMM_NCCL ? 0 : rank;
  if (!c->have[slot]) return fail(KTILER_E_STATE, "strip of rank " + std::to_string(rank) + " not registered");
  const ktiler_strip& s = c->strips[slot];
  const HaloRows R = halo_rows_of(s, rank, c->nranks, h);
  if (c->kind == KTILER_COMM_LOOPBACK) {
    // validate both neighbours before any copy is issued
    for (int nb : {rank - 1, rank + 1}) {
      if ((nb == rank - 1 && !R.recv_top) || (nb == rank + 1 && !R.recv_bot)) continue;
      if (!c->have[nb]) return fail(KTILER_E_STATE, "strip of rank " + std::to_string(nb) + " not registered");
    }
    // my halo rows are my neighbours' owned rows: one 2-D copy per halo
    if (R.recv_top) {
      if (!c->have[rank - 1]) return fail(KTILER_E_STATE, "strip of rank " + std::to_string(rank - 1) + " not registered");
      const ktiler_strip& u = c->strips[rank - 1];
      if (u.o1 != s.o0 || u.o1 - u.o0 < R.recv_top) return fail(KTILER_E_INVALID, "strips of ranks r-1, r do not abut");
      cudaError_t e = cudaMemcpy2DAsync(row_at(s, s.e0), s.pitch_bytes, row_at(u, u.o1 - R.recv_top), u.pitch_bytes,
                                        s.row_bytes, R.recv_top, cudaMemcpyDeviceToDevice, st);
      if (e != cudaSuccess) return fail(KTILER_E_CUDA, std::string("halo copy: ") + cudaGetErrorString(e));
    }
    if (R.recv_bot) {
      if (!c->have[rank + 1]) return fail(KTILER_E_STATE, "strip of rank " + std::to_string(rank + 1) + " not registered");
      const ktiler_strip& d = c->strips[rank + 1];
      if (d.o0 != s.o1 || d.o1 - d.o0 < R.recv_bot) return fail(KTILER_E_INVALID, "strips of ranks r, r+1 do not abut");
      cudaError_t e = cudaMemcpy2DAsync(row_at(s, s.o1), s.pitch_bytes, row_at(d, d.o0), d.pitch_bytes, s.row_bytes,
                                        R.recv_bot, cudaMemcpyDeviceToDevice, st);
      if (e != cudaSuccess) return fail(KTILER_E_CUDA, std::string("halo copy: ") + cudaGetErrorString(e));
    }
    return KTILER_OK;
  }
  // NCCL: contiguous row blocks (pitch x rows bytes; the pitch padding travels too)
  const NcclApi& a = nccl();
  if (!a.ok) return fail(KTILER_E_UNSUPPORTED, a.why);
  ncclResult_t r = a.GroupStart();
  if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
  const size_t pb = (size_t)s.pitch_bytes;
  if (R.recv_top) r = a.Recv(row_at(s, s.e0), pb * R.recv_top, ncclUint8, rank - 1, c->nc, st);
  if (r == ncclSuccess && R.send_up) r = a.Send(row_at(s, s.o0), pb * R.send_up, ncclUint8, rank - 1, c->nc, st);
  if (r == ncclSuccess && R.recv_bot) r = a.Recv(row_at(s, s.o1), pb * R.recv_bot, ncclUint8, rank + 1, c->nc, st);
  if (r == ncclSuccess && R.send_down)
    r = a.Send(row_at(s, s.o1 - R.send_down), pb * R.send_down, ncclUint8, rank + 1, c->nc, st);
  const ncclResult_t r2 = a.GroupEnd();
  if (r != ncclSuccess) return nccl_fail(r, "ncclSend/ncclRecv");
  if (r2 != ncclSuccess) return nccl_fail(r2, "ncclGroupEnd");
  return KTILER_OK;
}

}  // namespace kt

extern "C" {

ktiler_status ktiler_comm_unique_id(uint8_t* id128) {
  if (!id128) return fail(KTILER_E_INVALID, "NULL id");
  const NcclApi& a = nccl();
  if (!a.ok) return fail(KTILER_E_UNSUPPORTED, a.why);
  ncclUniqueId u;
  const ncclResult_t r = a.GetUniqueId(&u);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  static_assert(sizeof(u) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(id128, &u, 128);
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_comm_init_nccl(const uint8_t* id128, int32_t nranks, int32_t rank, ktiler_comm_t* out) {
  if (!id128 || !out || nranks < 1 || rank < 0 || rank >= nranks) return fail(KTILER_E_INVALID, "bad argument");
  *out = nullptr;
  const NcclApi& a = nccl();
  if (!a.ok) return fail(KTILER_E_UNSUPPORTED, a.why);
  ncclUniqueId u;
  std::memcpy(&u, id128, 128);
  auto* c = new ktiler_comm_s();
  c->kind = KTILER_COMM_NCCL;
  c->nranks = nranks;
  c->rank = rank;
  c->strips.resize(1);
  c->have.assign(1, 0);
  const ncclResult_t r = a.CommInitRank(&c->nc, nranks, u, rank);
  if (r != ncclSuccess) {
    c->nc = nullptr;
    delete c;
    return nccl_fail(r, "ncclCommInitRank");
  }
  *out = c;
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_comm_init_loopback(int32_t nranks, ktiler_comm_t* out) {
  if (!out || nranks < 1) return fail(KTILER_E_INVALID, "bad argument");
  auto* c = new ktiler_comm_s();
  c->kind = KTILER_COMM_LOOPBACK;
  c->nranks = nranks;
  c->strips.resize(nranks);
  c->have.assign(nranks, 0);
  *out = c;
  kt::clear_error();
  return KTILER_OK;
}

void ktiler_comm_destroy(ktiler_comm_t c) { delete c; }

ktiler_status ktiler_comm_register_strip(ktiler_comm_t c, int32_t rank, const ktiler_strip* s) {
  if (!c || !s || rank < 0 || rank >= c->nranks) return fail(KTILER_E_INVALID, "bad comm, rank or strip");
  if (c->kind == KTILER_COMM_NCCL && rank != c->rank) return fail(KTILER_E_INVALID, "NCCL comm: register this rank's strip");
  if (!s->base || s->row_bytes <= 0 || s->pitch_bytes < s->row_bytes || !(s->e0 <= s->o0 && s->o0 < s->o1 && s->o1 <= s->e1))
    return fail(KTILER_E_INVALID, "strip: need base, pitch >= row bytes and e0 <= o0 < o1 <= e1");
  const int slot = c->kind == KTILER_COMM_NCCL ? 0 : rank;
  c->strips[slot] = *s;
  c->have[slot] = 1;
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_comm_check(ktiler_comm_t c) {
  if (!c) return fail(KTILER_E_INVALID, "NULL comm");
  if (c->kind != KTILER_COMM_NCCL || !c->nc) {
    kt::clear_error();
    return KTILER_OK;
  }
  const NcclApi& a = nccl();
  if (!a.CommGetAsyncError) return fail(KTILER_E_UNSUPPORTED, "ncclCommGetAsyncError not available");
  ncclResult_t r = ncclSuccess;
  const ncclResult_t q = a.CommGetAsyncError(c->nc, &r);
  if (q != ncclSuccess) return nccl_fail(q, "ncclCommGetAsyncError");
  if (r != ncclSuccess && r != ncclInProgress) return nccl_fail(r, "NCCL communicator (asynchronous error)");
  kt::clear_error();
  return KTILER_OK;
}

ktiler_status ktiler_halo_exchange(ktiler_comm_t c, int32_t rank, int32_t halo_rows, void* stream) {
  ktiler_status s = kt::halo_exchange(c, rank, halo_rows, stream);
  if (!s) kt::clear_error();
  return s;
}

}  // extern "C"
