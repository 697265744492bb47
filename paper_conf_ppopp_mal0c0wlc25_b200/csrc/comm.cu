// comm.cu -- one process per GPU: peer-mapped buffers and the device barrier.
//
// The strategy kernels address other ranks' buffers only through device pointer
// tables (feature shards, requesters' h^1 / g, owners' work lists, gradient
// buffers).  In a job of one process per GPU those tables hold CUDA-IPC-mapped
// peer pointers: loads, stores and atomics then travel over NVLink / NVSwitch
// directly from the kernels (the peer-store Reshuffle epilogue, the halo reads of
// GDP/DNP, the all-reduce).  Handles are exchanged once, at object creation,
// through a caller-supplied all-gather (apt_ctx_set_exchange: torch.distributed
// in the Python binding) -- bootstrap plumbing only, never on the step path.
// Phases of a step are separated by a device-side flag barrier (graph-capturable,
// no host round trip): every rank release-stores its epoch into a slot of every
// peer's flag array, then acquire-spins until all C slots of its own array reach
// the epoch.
#include <cstring>
#include <vector>

#include "common.cuh"
#include "runtime.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
apt_status check_cuda(apt_ctx* c, cudaError_t e, const char* what);

bool multiprocess(const apt_ctx* c) { return c && !c->emulated && c->world > 1; }

apt_status allgather(apt_ctx* c, const void* send, void* recv, size_t bytes) {
  if (!c->exchange) return set_err(c, APT_E_STATE, "multi-process ctx: call apt_ctx_set_exchange first");
  if (c->exchange(send, recv, bytes, c->exchange_user) != 0)
    return set_err(c, APT_E_COMM, "exchange callback failed");
  return APT_OK;
}

// tab[p] = rank p's `local` allocation (opened through IPC), tab[rank] = local.
apt_status share_ptr(apt_ctx* c, void* local, void** tab, std::vector<void*>* opened) {
  if (!multiprocess(c)) return set_err(c, APT_E_STATE, "share_ptr: not a multi-process ctx");
  cudaIpcMemHandle_t mine;
  memset(&mine, 0, sizeof mine);
  cudaError_t e = cudaIpcGetMemHandle(&mine, local);
  if (e != cudaSuccess) return check_cuda(c, e, "cudaIpcGetMemHandle");
  std::vector<cudaIpcMemHandle_t> all(c->world);
  apt_status s = allgather(c, &mine, all.data(), sizeof mine);
  if (s != APT_OK) return s;
  for (int p = 0; p < c->world; ++p) {
    if (p == c->rank) { tab[p] = local; continue; }
    void* q = nullptr;
    e = cudaIpcOpenMemHandle(&q, all[p], cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return check_cuda(c, e, "cudaIpcOpenMemHandle");
    tab[p] = q;
    if (opened) opened->push_back(q);
  }
  return APT_OK;
}

void close_peers(std::vector<void*>& opened) {
  for (void* p : opened) cudaIpcCloseMemHandle(p);
  opened.clear();
}

void defer_exported(apt_ctx* c, Arena& a) {
  if (!multiprocess(c)) return;
  cudaStreamSynchronize(c->stream);
  for (auto& b : a.bufs) c->deferred.push_back(b);
  a.bufs.clear();
  a.total = 0;
}

// ctx teardown in a multi-process job: close every mapping, wait for all peers to
// have done the same (host all-gather), then free what this rank exported.
void release_exported(apt_ctx* c) {
  close_peers(c->peer_opened);
  if (multiprocess(c) && c->exchange) {
    char x = 0;
    std::vector<char> all(c->world);
    c->exchange(&x, all.data(), 1, c->exchange_user);   // best effort at interpreter exit
  }
  for (auto& b : c->deferred) cudaFree(b.p);
  c->deferred.clear();
}

// ---------------------------------------------------------------- barrier
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__global__ void barrier_kernel(uint64_t* const* flags, uint64_t* my_flags, uint64_t* epoch, int rank, int C,
                               uint32_t* err) {
  APT_PDL_PROLOGUE();
  if (threadIdx.x != 0) return;
  const uint64_t e = *epoch + 1;
  *epoch = e;
  __threadfence_system();
  for (int p = 0; p < C; ++p) st_release_sys(flags[p] + rank, e);
  const uint64_t t0 = globaltimer();
  for (int q = 0; q < C; ++q) {
    while (ld_acquire_sys(my_flags + q) < e) {
      if (globaltimer() - t0 > 30ull * 1000000000ull) {   // a peer never arrived: fail, do not hang
        atomicOr(err, kDevErrTimeout);
        return;
      }
      __nanosleep(64);
    }
  }
}

apt_status barrier_setup(apt_ctx* c) {
  if (!multiprocess(c) || c->bar_tab) return APT_OK;
  c->bar_flags = c->arena.alloc<uint64_t>(APT_MAX_RANKS + 1, true);   // [C] slots + the epoch
  if (!c->bar_flags) return set_err(c, APT_E_OOM, "barrier_setup: out of device memory");
  void* tab[APT_MAX_RANKS] = {};
  apt_status s = share_ptr(c, c->bar_flags, tab, &c->peer_opened);
  if (s != APT_OK) return s;
  c->bar_tab = c->arena.alloc<uint64_t*>(c->world, false);
  if (!c->bar_tab) return set_err(c, APT_E_OOM, "barrier_setup: out of device memory");
  cudaError_t e = cudaMemcpy(c->bar_tab, tab, sizeof(void*) * c->world, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return check_cuda(c, e, "barrier_setup");
  // every rank's flags must exist before anyone can signal: one host-side sync point
  char x = 0;
  std::vector<char> all(c->world);
  return allgather(c, &x, all.data(), 1);
}

apt_status device_barrier(apt_ctx* c) {
  if (!multiprocess(c)) return APT_OK;
  if (!c->bar_tab) return set_err(c, APT_E_STATE, "device_barrier: barrier not set up");
  launch_pdl(barrier_kernel, dim3(1), dim3(32), 0, c->stream, c->bar_tab, c->bar_flags, c->bar_flags + APT_MAX_RANKS, c->rank, c->world,
                                          c->dev_err);
  c->launches++;
  return check_cuda(c, cudaGetLastError(), "barrier_kernel");
}

}  // namespace apt

using namespace apt;

extern "C" {

apt_status apt_ctx_set_exchange(apt_ctx* c, apt_allgather_fn fn, void* user) {
  if (!c || !fn) return set_err(c, APT_E_INVALID, "apt_ctx_set_exchange: bad arguments");
  c->exchange = fn;
  c->exchange_user = user;
  return barrier_setup(c);
}

// Host-only check of the exchange protocol (no GPU needed): every rank sends
// `bytes` bytes of the pattern (rank, i) and checks that recv holds every rank's
// block in rank order.
apt_status apt_exchange_selftest(int rank, int world, apt_allgather_fn fn, void* user) {
  if (!fn || world < 1 || rank < 0 || rank >= world) return set_err(nullptr, APT_E_INVALID, "apt_exchange_selftest: bad args");
  const size_t bytes = 64 + 7;   // odd size: like a cudaIpcMemHandle_t plus framing
  std::vector<unsigned char> send(bytes), recv(bytes * world, 0xEE);
  for (size_t i = 0; i < bytes; ++i) send[i] = (unsigned char)(rank * 31 + i * 7);
  if (fn(send.data(), recv.data(), bytes, user) != 0) return set_err(nullptr, APT_E_COMM, "exchange callback failed");
  for (int p = 0; p < world; ++p)
    for (size_t i = 0; i < bytes; ++i)
      if (recv[p * bytes + i] != (unsigned char)(p * 31 + i * 7))
        return set_err(nullptr, APT_E_COMM, "exchange: rank %d byte %zu wrong", p, i);
  return APT_OK;
}

}  // extern "C"
