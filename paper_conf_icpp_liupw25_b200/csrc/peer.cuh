// peer.cuh — fused peer-memory exchange of the feature-partitioned multi-GPU scheme (
// SURVEY §8(f) NEXT-4).  Every rank owns one "window" of device memory that all ranks map (CUDA IPC
// over NVLink / NVSwitch); the per-level exchanges become loads from the peers' windows inside the
// kernels that consume them, with a flag per phase instead of a host-issued collective:
//
//   find_split / search_small  write this rank's keys into its own window (no copy)
//   split_record   prologue:   publish flag_keys = E, wait until every peer's flag_keys >= E,
//                              key[slot] = max over the N windows (the MAX all-reduce)
//                  body:       owner's records + bitmap into its own window (no copy)
//   partition      prologue:   publish flag_rec = E, wait, xchg = sum over the N windows (the SUM
//                              all-reduce: non-owners hold zeros, bitmap bits are disjoint)
//
// E = epoch + 1, epoch = exchanges completed (a device word of the own window, incremented by the
// partition's plan kernel), identical on every rank since all run the same sequence; CUDA graphs
// replay correctly because nothing host-side carries the epoch.  A rank rewrites its keys only
// after every peer published flag_rec (so finished reading them) and its records only after every
// peer published the next flag_keys; one buffer per kind would be race-free, per-level buffers are
// kept for debugging (model-checked: tests/test_peer_protocol.py).
// Waits are bounded (GBDTMO_OPT_PEER_TIMEOUT_MS): on expiry the kernel records an error word
// (gbdtmo_peer_status) and proceeds, so a lost peer cannot hang the GPU.
#pragma once

#include "common.cuh"

namespace gbdtmo {

constexpr int kPeerMax = 8;
// header words (uint64) of a window; flags 128 bytes apart
enum { PEER_FLAG_KEYS = 0, PEER_FLAG_REC = 16, PEER_EPOCH = 32, PEER_ERROR = 48, PEER_HEADER_WORDS = 64 };

struct PeerView {
  char* win[kPeerMax];   // window base of every rank (own one included), device pointers
  int32_t world;         // 0: no peer exchange
  int32_t rank;
  int64_t timeout_ns;
};

// Window layout: header, then keys [D][2^(D-1)] uint64, then xchg [D][xchg_count] int64.
__host__ __device__ inline int64_t peer_xchg_count(const gbdtmo_problem& p) { return bitmap_offset(p) + (p.n + 63) / 64; }
__host__ __device__ inline int64_t peer_keys_off(const gbdtmo_problem& p, int level) {
  return 8 * PEER_HEADER_WORDS + 8 * (int64_t)level * max_level_nodes(p);
}
__host__ __device__ inline int64_t peer_xchg_off(const gbdtmo_problem& p, int level) {
  const int64_t k = (int64_t)align_up((size_t)peer_keys_off(p, p.D), 256);
  return k + 8 * (int64_t)level * (int64_t)align_up((size_t)peer_xchg_count(p), 32);
}
__host__ __device__ inline int64_t peer_window_bytes(const gbdtmo_problem& p) { return peer_xchg_off(p, p.D); }

__device__ __forceinline__ uint64_t peer_ld_acquire(const uint64_t* a) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(a) : "memory");
  return v;
}
__device__ __forceinline__ void peer_st_release(uint64_t* a, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(a), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t peer_clock_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint64_t* peer_word(const PeerView& pv, int r, int w) {
  return reinterpret_cast<uint64_t*>(pv.win[r]) + w;
}

// This exchange's epoch value (read at kernel start; only the plan kernel of the partition,
// which runs after both phases of a level, changes it).
__device__ __forceinline__ uint64_t peer_next_epoch(const PeerView& pv) {
  return *reinterpret_cast<volatile uint64_t*>(peer_word(pv, pv.rank, PEER_EPOCH)) + 1;
}

// Called by one thread.  publish: store flag = E on the own window after the writes this rank
// made to it (earlier kernels on the stream) — release at system scope.  Then wait for every peer.
__device__ inline bool peer_publish_wait(const PeerView& pv, int flag, uint64_t E, bool publish) {
  if (publish) {
    __threadfence_system();
    peer_st_release(peer_word(pv, pv.rank, flag), E);
  }
  // a previous wait already expired: fail fast (outputs are invalid anyway; no second timeout)
  if (*reinterpret_cast<volatile uint64_t*>(peer_word(pv, pv.rank, PEER_ERROR)) != 0) return false;
  const uint64_t t0 = peer_clock_ns();
  for (int r = 0; r < pv.world; ++r) {
    if (r == pv.rank) continue;
    const uint64_t* f = peer_word(pv, r, flag);
    while (peer_ld_acquire(f) < E) {
      if (peer_clock_ns() - t0 > (uint64_t)pv.timeout_ns) {
        __threadfence_system();
        atomicCAS(reinterpret_cast<unsigned long long*>(peer_word(pv, pv.rank, PEER_ERROR)), 0ull,
                  (unsigned long long)(E << 8 | (uint64_t)(flag == PEER_FLAG_KEYS ? 1 : 2)));
        return false;
      }
      __nanosleep(128);
    }
  }
  // a peer that failed earlier has diverged (its nodes became leaves): adopt its failure, so this
  // rank stops splitting too instead of partitioning from records of a different tree.  The
  // peer's error store precedes its flag store (fence), so the acquire above makes it visible.
  for (int r = 0; r < pv.world; ++r) {
    if (r == pv.rank) continue;
    const uint64_t e = peer_ld_acquire(peer_word(pv, r, PEER_ERROR));
    if (e) {
      atomicCAS(reinterpret_cast<unsigned long long*>(peer_word(pv, pv.rank, PEER_ERROR)), 0ull,
                (unsigned long long)e);
      return false;
    }
  }
  return true;
}

// Peer data is read with ld.global.cv (no L1/L2 caching of another GPU's lines).
__device__ __forceinline__ uint64_t peer_load(const uint64_t* a) {
  return (uint64_t)__ldcv(reinterpret_cast<const unsigned long long*>(a));
}

// Host side: the context's peer group (peer.cu).
struct Peer;
PeerView peer_view(const Ctx* ctx);
bool peer_ready(const Ctx* ctx, const gbdtmo_problem& p);
char* peer_own_window(const Ctx* ctx);
void peer_release(Ctx* ctx);
// Fused gather of a level's records + bitmap from every window into xchg_out (k_peer_gather).
gbdtmo_status peer_gather(Ctx* ctx, const gbdtmo_problem& p, int level, int64_t* xchg_out);

}  // namespace gbdtmo
