// peer.cu — NEXT-4 ("partial histograms ... aggregated across GPUs"):
// lifecycle of the peer-memory exchange group and the fused gather of the split records.
// Protocol and layout: peer.cuh.  The windows are plain cudaMalloc allocations exported with CUDA
// IPC; on an NVSwitch box a peer's window is reached over NVLink with ordinary loads.
#include <string.h>

#include <new>

#include "peer.cuh"

namespace gbdtmo {

struct Peer {
  int rank = 0, world = 0;
  gbdtmo_problem shape{};      // the problem the window was sized for
  size_t bytes = 0;
  char* own = nullptr;         // this rank's window (cudaMalloc)
  char* win[kPeerMax] = {};    // every rank's window as mapped here (win[rank] = own)
  bool connected = false;
};

PeerView peer_view(const Ctx* ctx) {
  PeerView v;
  memset(&v, 0, sizeof(v));
  const Peer* pr = ctx->peer;
  if (!pr || !pr->connected) return v;
  for (int r = 0; r < pr->world; ++r) v.win[r] = pr->win[r];
  v.world = pr->world;
  v.rank = pr->rank;
  v.timeout_ns = ctx->peer_timeout_ms * 1000000ll;
  return v;
}

static bool same_shape(const gbdtmo_problem& a, const gbdtmo_problem& b) {
  return a.n == b.n && a.D == b.D && channels(a) == channels(b);
}

bool peer_ready(const Ctx* ctx, const gbdtmo_problem& p) {
  return ctx->peer && ctx->peer->connected && same_shape(ctx->peer->shape, p);
}

char* peer_own_window(const Ctx* ctx) { return ctx->peer ? ctx->peer->own : nullptr; }

void peer_release(Ctx* ctx) {
  Peer* pr = ctx->peer;
  if (!pr) return;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(ctx->device);
  cudaDeviceSynchronize();
  for (int r = 0; r < pr->world; ++r)
    if (pr->win[r] && pr->win[r] != pr->own) cudaIpcCloseMemHandle(pr->win[r]);
  if (pr->own) cudaFree(pr->own);
  cudaGetLastError();
  cudaSetDevice(prev);
  delete pr;
  ctx->peer = nullptr;
}

// Fused gather of the level's split records and bitmap (the SUM all-reduce): publish flag_rec,
// wait for every peer, then xchg_out[i] = sum over ranks of window_r.xchg[level][i] with 16-byte
// loads from the N windows.
__global__ void __launch_bounds__(256)
k_peer_gather(gbdtmo_problem p, int level, PeerView pv, int64_t* __restrict__ xchg_out) {
  __shared__ int ok;
  if (threadIdx.x == 0) {
    const uint64_t E = peer_next_epoch(pv);
    ok = peer_publish_wait(pv, PEER_FLAG_REC, E, blockIdx.x == 0);
  }
  __syncthreads();
  const int64_t total = peer_xchg_count(p), off = peer_xchg_off(p, level) / 8;
  const int64_t pairs = total / 2;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  if (!ok) {          // an expired wait (error word set): no records, every node of the level stays a leaf
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += stride) xchg_out[i] = 0;
    return;
  }
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < pairs; i += stride) {
    long long a = 0, b = 0;
    for (int r = 0; r < pv.world; ++r) {
      const longlong2 v = __ldcv(reinterpret_cast<const longlong2*>(reinterpret_cast<int64_t*>(pv.win[r]) + off) + i);
      a += v.x;
      b += v.y;
    }
    reinterpret_cast<longlong2*>(xchg_out)[i] = make_longlong2(a, b);
  }
  if ((total & 1) && blockIdx.x == 0 && threadIdx.x == 0) {
    long long a = 0;
    for (int r = 0; r < pv.world; ++r)
      a += (long long)peer_load(reinterpret_cast<const uint64_t*>(pv.win[r]) + off + total - 1);
    xchg_out[total - 1] = a;
  }
}

gbdtmo_status peer_gather(Ctx* ctx, const gbdtmo_problem& p, int level, int64_t* xchg_out) {
  const PeerView pv = peer_view(ctx);
  const int64_t pairs = peer_xchg_count(p) / 2;
  int grid = (int)((pairs + 255) / 256);
  grid = grid < 1 ? 1 : grid > 2 * ctx->num_sms ? 2 * ctx->num_sms : grid;
  GB_LAUNCH(k_peer_gather, grid, 256, 0, p, level, pv, xchg_out);
  return GBDTMO_OK;
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" size_t gbdtmo_peer_window_bytes(const gbdtmo_problem* p) {
  if (check_problem(p)) return 0;
  return (size_t)peer_window_bytes(*p);
}

extern "C" gbdtmo_status gbdtmo_peer_open(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t rank, int32_t world,
                                          uint8_t* handle) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(handle, "null handle buffer");
  GB_CHECK_ARG(world >= 1 && world <= kPeerMax, "world out of range [1, 8]");
  GB_CHECK_ARG(rank >= 0 && rank < world, "rank out of range [0, world)");
  peer_release(ctx);
  Peer* pr = new (std::nothrow) Peer();
  if (!pr) return GBDTMO_ENOMEM;
  pr->rank = rank;
  pr->world = world;
  pr->shape = *p;
  pr->bytes = (size_t)peer_window_bytes(*p);
  cudaIpcMemHandle_t h;
  if (cudaMalloc(&pr->own, pr->bytes) != cudaSuccess || cudaMemset(pr->own, 0, pr->bytes) != cudaSuccess ||
      cudaDeviceSynchronize() != cudaSuccess || cudaIpcGetMemHandle(&h, pr->own) != cudaSuccess) {
    ctx->err = std::string("gbdtmo_peer_open: ") + cudaGetErrorString(cudaGetLastError());
    if (pr->own) cudaFree(pr->own);
    delete pr;
    return GBDTMO_ECUDA;
  }
  static_assert(sizeof(cudaIpcMemHandle_t) == GBDTMO_PEER_HANDLE_BYTES, "IPC handle size");
  memcpy(handle, &h, sizeof(h));
  pr->win[rank] = pr->own;
  ctx->peer = pr;
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_peer_connect(gbdtmo_ctx c, const uint8_t* handles) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(ctx->peer, "gbdtmo_peer_open first");
  GB_CHECK_ARG(handles, "null handles");
  Peer* pr = ctx->peer;
  GB_CHECK_ARG(!pr->connected, "already connected");
  for (int r = 0; r < pr->world; ++r) {
    if (r == pr->rank) continue;
    cudaIpcMemHandle_t h;
    memcpy(&h, handles + (size_t)r * GBDTMO_PEER_HANDLE_BYTES, sizeof(h));
    void* ptr = nullptr;
    if (cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
      ctx->err = std::string("gbdtmo_peer_connect: rank ") + std::to_string(r) + ": " +
                 cudaGetErrorString(cudaGetLastError());
      for (int q = 0; q < r; ++q)
        if (q != pr->rank && pr->win[q]) { cudaIpcCloseMemHandle(pr->win[q]); pr->win[q] = nullptr; }
      return GBDTMO_ECUDA;
    }
    pr->win[r] = (char*)ptr;
  }
  pr->connected = true;
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_peer_buffers(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level, uint64_t** keys,
                                             int64_t** xchg) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(ctx->peer && same_shape(ctx->peer->shape, *p), "no peer window for this problem shape");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  if (keys) *keys = reinterpret_cast<uint64_t*>(ctx->peer->own + peer_keys_off(*p, level));
  if (xchg) *xchg = reinterpret_cast<int64_t*>(ctx->peer->own + peer_xchg_off(*p, level));
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_peer_status(gbdtmo_ctx c, int64_t* epoch, int64_t* error) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(ctx->peer, "no peer window");
  uint64_t hdr[PEER_HEADER_WORDS];
  if (cudaMemcpy(hdr, ctx->peer->own, sizeof(hdr), cudaMemcpyDeviceToHost) != cudaSuccess) {
    ctx->err = std::string("gbdtmo_peer_status: ") + cudaGetErrorString(cudaGetLastError());
    return GBDTMO_ECUDA;
  }
  if (epoch) *epoch = (int64_t)hdr[PEER_EPOCH];
  if (error) *error = (int64_t)hdr[PEER_ERROR];
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_peer_status_async(gbdtmo_ctx c, int64_t* out) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(ctx->peer, "no peer window");
  GB_CHECK_ARG(out, "null output");
  const uint64_t* hdr = reinterpret_cast<const uint64_t*>(ctx->peer->own);
  if (cudaMemcpyAsync(out, hdr + PEER_EPOCH, 8, cudaMemcpyDefault, ctx->stream) != cudaSuccess ||
      cudaMemcpyAsync(out + 1, hdr + PEER_ERROR, 8, cudaMemcpyDefault, ctx->stream) != cudaSuccess) {
    ctx->err = std::string("gbdtmo_peer_status_async: ") + cudaGetErrorString(cudaGetLastError());
    return GBDTMO_ECUDA;
  }
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_peer_close(gbdtmo_ctx c) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  peer_release(ctx);
  return GBDTMO_OK;
}
