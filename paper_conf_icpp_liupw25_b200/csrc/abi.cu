// abi.cu — context lifecycle and size queries of the C ABI (include/gbdtmo.h).
#include <new>

#include "common.cuh"
#include "peer.cuh"

using namespace gbdtmo;

extern "C" int gbdtmo_abi_version(void) { return GBDTMO_ABI_VERSION; }

extern "C" gbdtmo_status gbdtmo_create(int device, gbdtmo_ctx* out) {
  if (!out) return GBDTMO_EINVAL;
  *out = nullptr;
  int count = 0;
  if (cudaGetDeviceCount(&count) != cudaSuccess || device < 0 || device >= count) {
    cudaGetLastError();
    return GBDTMO_ECUDA;
  }
  Ctx* ctx = new (std::nothrow) Ctx();
  if (!ctx) return GBDTMO_ENOMEM;
  ctx->device = device;
  GB_ENTRY(ctx);          // restores the caller's device on return
  if (cudaGetLastError() != cudaSuccess ||
      cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess ||
      cudaDeviceGetAttribute(&ctx->max_smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device) != cudaSuccess) {
    cudaGetLastError();
    delete ctx;
    return GBDTMO_ECUDA;
  }
  *out = (gbdtmo_ctx)ctx;
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_destroy(gbdtmo_ctx c) {
  if (c) {
    peer_release((Ctx*)c);
    ctx_release_streams((Ctx*)c);
  }
  delete (Ctx*)c;
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_set_stream(gbdtmo_ctx c, void* stream) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  ctx->stream = (cudaStream_t)stream;
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_set_option(gbdtmo_ctx c, int32_t option, int64_t value) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  switch (option) {
    case GBDTMO_OPT_GMEM_MAX_ROWS: ctx->gmem_max_rows = value; return GBDTMO_OK;
    case GBDTMO_OPT_SMALL_MAX_ROWS: ctx->small_max_rows = value; return GBDTMO_OK;
    case GBDTMO_OPT_HIST_KERNEL:
      if (value < 0 || value > 2) { ctx->err = "gbdtmo_set_option: HIST_KERNEL must be 0, 1 or 2"; return GBDTMO_EINVAL; }
      ctx->hist_kernel = value;
      return GBDTMO_OK;
    case GBDTMO_OPT_PEER_TIMEOUT_MS:
      if (value < 1) { ctx->err = "gbdtmo_set_option: PEER_TIMEOUT_MS must be >= 1"; return GBDTMO_EINVAL; }
      ctx->peer_timeout_ms = value;
      return GBDTMO_OK;
    case GBDTMO_OPT_FS_CHANNEL_GROUPS:
      if (value != 0 && value != 1 && value != 2 && value != 4 && value != 8) {
        ctx->err = "gbdtmo_set_option: FS_CHANNEL_GROUPS must be 0, 1, 2, 4 or 8";
        return GBDTMO_EINVAL;
      }
      ctx->fs_channel_groups = value;
      return GBDTMO_OK;
    case GBDTMO_OPT_HIST_WAVES:
      if (value < 0 || value > 64) { ctx->err = "gbdtmo_set_option: HIST_WAVES must be in [0, 64]"; return GBDTMO_EINVAL; }
      ctx->hist_waves = value;
      return GBDTMO_OK;
    default: ctx->err = "gbdtmo_set_option: unknown option"; return GBDTMO_EINVAL;
  }
}

extern "C" const char* gbdtmo_last_error(gbdtmo_ctx c) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  return ctx ? ctx->err.c_str() : "null context";
}

extern "C" int64_t gbdtmo_launch_count(gbdtmo_ctx c) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  return ctx ? ctx->launches : -1;
}

extern "C" size_t gbdtmo_bins_bytes(int64_t n, int64_t ld_bins) { return (size_t)(n * ld_bins + 32); }

extern "C" gbdtmo_status gbdtmo_state_bytes(const gbdtmo_problem* p, size_t* bytes) {
  if (!bytes || check_problem(p)) return GBDTMO_EINVAL;
  *bytes = state_layout(*p).total;
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_hist_bytes(const gbdtmo_problem* p, int32_t level, size_t* hist_bytes,
                                           size_t* cnt_bytes) {
  if (check_problem(p) || level < 0 || level >= p->D) return GBDTMO_EINVAL;
  const size_t LN = (size_t)hist_slots(*p, level);
  if (hist_bytes) *hist_bytes = LN * (size_t)p->m * p->B * channels(*p) * 8;
  if (cnt_bytes) *cnt_bytes = LN * (size_t)p->m * p->B * 4;
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_xchg_count(const gbdtmo_problem* p, int64_t* count) {
  if (!count || check_problem(p)) return GBDTMO_EINVAL;
  *count = bitmap_offset(*p) + (p->n + 63) / 64;
  return GBDTMO_OK;
}
