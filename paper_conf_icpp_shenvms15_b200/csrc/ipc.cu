// Multi-process transport: shared-memory rendezvous + CUDA IPC flags (ipc.h).
#include <cuda.h>
#include <fcntl.h>
#include <sched.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <functional>
#include <thread>

#include "ipc.h"
#include "kernels.h"
#include "mm_internal.h"

namespace mm {

namespace {

constexpr uint32_t kMagic = 0x6d6d4950u;   // "mmIP"
constexpr double kTimeoutS = 120.0;

template <class T>
T ld_acq(T* p) { return __atomic_load_n(p, __ATOMIC_ACQUIRE); }
template <class T>
void st_rel(T* p, T v) { __atomic_store_n(p, v, __ATOMIC_RELEASE); }

bool spin_until(const std::function<bool()>& ok, const ShmBlock* shm) {
  const auto t0 = std::chrono::steady_clock::now();
  for (uint64_t i = 0;; ++i) {
    if (ok()) return true;
    if (shm && __atomic_load_n(&shm->failed, __ATOMIC_ACQUIRE)) return false;
    if (i > 1000) {
      if (i % 64 == 0 &&
          std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > kTimeoutS)
        return false;
      sched_yield();
    }
  }
}

using GetRangeFn = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
GetRangeFn get_range() {
  static GetRangeFn fn = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return (GetRangeFn) nullptr;
    return (GetRangeFn)p;
  }();
  return fn;
}

std::string key_of(const cudaIpcMemHandle_t& h) { return std::string(h.reserved, sizeof(h.reserved)); }

// ---------------------------------------------------------------- kernels --
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__global__ void k_bump(uint64_t* flags) { flags[kIpcEpoch] += 1; }

__global__ void k_signal(uint64_t* flags, int64_t slot) {
  const uint64_t e = flags[kIpcEpoch];
  __threadfence_system();
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(flags + slot), "l"(e) : "memory");
}

struct WaitArgs {
  const uint64_t* f[8];
  uint32_t lag[8];
};

__global__ void k_wait(const uint64_t* my, WaitArgs a, int n) {
  const int i = threadIdx.x;
  if (i >= n) return;
  const uint64_t target = my[kIpcEpoch] - a.lag[i];
  uint64_t t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  while (ld_acquire_sys(a.f[i]) < target) {
    __nanosleep(200);
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 60ull * 1000000000ull) __trap();   // a peer never signalled: fail, never hang
  }
}

}  // namespace

cudaError_t ipc_bump_epoch(uint64_t* flags, cudaStream_t s) {
  note_launch();
  k_bump<<<1, 1, 0, s>>>(flags);
  return cudaGetLastError();
}

cudaError_t ipc_signal(uint64_t* flags, int64_t slot, cudaStream_t s) {
  note_launch();
  k_signal<<<1, 1, 0, s>>>(flags, slot);
  return cudaGetLastError();
}

cudaError_t ipc_wait(const uint64_t* my_flags, uint64_t* const* peer, const int64_t* slot, const uint32_t* lag,
                     int32_t n, cudaStream_t s) {
  for (int32_t b = 0; b < n; b += 8) {
    WaitArgs a{};
    const int m = n - b < 8 ? n - b : 8;
    for (int i = 0; i < m; ++i) {
      a.f[i] = peer[b + i] + slot[b + i];
      a.lag[i] = lag[b + i];
    }
    note_launch();
    k_wait<<<1, 32, 0, s>>>(my_flags, a, m);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// ------------------------------------------------------------------- host --
mm_status ipc_barrier(IpcChannel* ch) {
  ShmBlock* s = ch->shm;
  const uint32_t gen = ld_acq(&s->bar_gen);
  if (__atomic_add_fetch(&s->bar_count, 1u, __ATOMIC_ACQ_REL) == (uint32_t)ch->world) {
    st_rel(&s->bar_count, 0u);
    st_rel(&s->bar_gen, gen + 1);
    return MM_OK;
  }
  if (!spin_until([&] { return ld_acq(&s->bar_gen) != gen; }, s)) {
    __atomic_store_n(&s->failed, 1, __ATOMIC_RELEASE);
    MM_FAIL(MM_ESTATE, "ipc: host barrier timed out (rank %d of %d)", ch->rank, ch->world);
  }
  return MM_OK;
}

mm_status ipc_open(IpcChannel* ch, const void* id128, int32_t rank, int32_t world) {
  ch->rank = rank;
  ch->world = world;
  const unsigned char* id = static_cast<const unsigned char*>(id128);
  char nm[64];
  int p = snprintf(nm, sizeof(nm), "/mm_rdv_");
  for (int i = 0; i < 12; ++i) p += snprintf(nm + p, sizeof(nm) - p, "%02x", id[i]);
  ch->name = nm;
  int fd = -1;
  if (rank == 0) {
    shm_unlink(nm);
    fd = shm_open(nm, O_CREAT | O_EXCL | O_RDWR, 0600);
    if (fd < 0) MM_FAIL(MM_ESTATE, "ipc: shm_open(%s) failed", nm);
    if (ftruncate(fd, sizeof(ShmBlock)) != 0) {
      close(fd);
      MM_FAIL(MM_ESTATE, "ipc: ftruncate failed");
    }
  } else {
    const bool ok = spin_until([&] { return (fd = shm_open(nm, O_RDWR, 0600)) >= 0; }, nullptr);
    if (!ok) MM_FAIL(MM_ESTATE, "ipc: rank %d: rendezvous %s not created by rank 0", rank, nm);
    struct stat st;
    if (!spin_until([&] { return fstat(fd, &st) == 0 && st.st_size >= (off_t)sizeof(ShmBlock); }, nullptr)) {
      close(fd);
      MM_FAIL(MM_ESTATE, "ipc: rendezvous block never sized");
    }
  }
  void* m = mmap(nullptr, sizeof(ShmBlock), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (m == MAP_FAILED) MM_FAIL(MM_ESTATE, "ipc: mmap failed");
  ch->shm = static_cast<ShmBlock*>(m);
  ShmBlock* s = ch->shm;
  if (rank == 0) {
    s->world = world;
    st_rel(&s->magic, kMagic);
  } else if (!spin_until([&] { return ld_acq(&s->magic) == kMagic; }, nullptr)) {
    MM_FAIL(MM_ESTATE, "ipc: rendezvous block never initialised");
  }
  if (s->world != world) MM_FAIL(MM_EINVAL, "ipc: world %d, rendezvous has %d", world, s->world);
  // flags on this rank's device
  if (cudaMalloc(&ch->flags, kIpcFlagSlots * sizeof(uint64_t)) != cudaSuccess)
    MM_FAIL(MM_ENOMEM, "ipc: flags");
  if (cudaMemset(ch->flags, 0, kIpcFlagSlots * sizeof(uint64_t)) != cudaSuccess ||
      cudaDeviceSynchronize() != cudaSuccess)
    MM_FAIL(MM_ECUDA, "ipc: flag init");
  if (cudaIpcGetMemHandle(&s->r[rank].flags_h, ch->flags) != cudaSuccess)
    MM_FAIL(MM_ECUDA, "ipc: flag handle");
  s->r[rank].pid = (uint64_t)getpid();
  __atomic_add_fetch(&s->attached, 1, __ATOMIC_ACQ_REL);
  mm_status st = ipc_barrier(ch);
  if (st) return st;
  if (rank == 0) shm_unlink(nm);   // every rank has it mapped
  ch->peer_flags.assign(world, nullptr);
  for (int32_t q = 0; q < world; ++q) {
    if (q == rank) {
      ch->peer_flags[q] = ch->flags;
      continue;
    }
    void* pf = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&pf, s->r[q].flags_h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) MM_FAIL(MM_ECUDA, "ipc: open flags of rank %d: %s", q, cudaGetErrorString(e));
    ch->peer_flags[q] = static_cast<uint64_t*>(pf);
  }
  return ipc_barrier(ch);
}

void ipc_close(IpcChannel* ch) {
  if (!ch) return;
  for (int32_t q = 0; q < (int32_t)ch->peer_flags.size(); ++q)
    if (q != ch->rank && ch->peer_flags[q]) cudaIpcCloseMemHandle(ch->peer_flags[q]);
  for (auto& kv : ch->opened) cudaIpcCloseMemHandle(kv.second);
  ch->opened.clear();
  if (ch->flags) cudaFree(ch->flags);
  if (ch->shm) munmap(ch->shm, sizeof(ShmBlock));
  ch->shm = nullptr;
  ch->flags = nullptr;
}

mm_status ipc_exchange_buffers(IpcChannel* ch, const std::vector<void*>& mine, std::vector<char*>& out) {
  const int32_t nb = (int32_t)mine.size();
  if (nb > MM_MAX_BUF) MM_FAIL(MM_EINVAL, "ipc: %d buffers", nb);
  const int par = (int)(ch->xchg++ & 1);
  ShmRank& me = ch->shm->r[ch->rank];
  for (int32_t b = 0; b < nb; ++b) {
    me.buf_null[par][b] = mine[b] == nullptr;
    if (!mine[b]) continue;
    auto it = ch->exported.find(mine[b]);
    if (it == ch->exported.end()) {
      GetRangeFn gr = get_range();
      if (!gr) MM_FAIL(MM_ENOTSUP, "ipc: cuMemGetAddressRange unavailable");
      CUdeviceptr base = 0;
      size_t sz = 0;
      if (gr(&base, &sz, (CUdeviceptr)mine[b]) != CUDA_SUCCESS) MM_FAIL(MM_EINVAL, "ipc: buffer %d not device memory", b);
      cudaIpcMemHandle_t h;
      cudaError_t e = cudaIpcGetMemHandle(&h, (void*)base);
      if (e != cudaSuccess) MM_FAIL(MM_ECUDA, "ipc: handle of buffer %d: %s", b, cudaGetErrorString(e));
      it = ch->exported.emplace(mine[b], std::make_pair(h, (uint64_t)((const char*)mine[b] - (const char*)base))).first;
    }
    me.buf_h[par][b] = it->second.first;
    me.buf_off[par][b] = it->second.second;
  }
  me.nbuf[par] = nb;
  mm_status st = ipc_barrier(ch);
  if (st) return st;
  out.assign((size_t)nb * ch->world, nullptr);
  for (int32_t q = 0; q < ch->world; ++q) {
    const ShmRank& r = ch->shm->r[q];
    if (r.nbuf[par] != nb) MM_FAIL(MM_EINVAL, "ipc: rank %d has %d buffers, rank %d has %d", q, r.nbuf[par], ch->rank, nb);
    for (int32_t b = 0; b < nb; ++b) {
      if (q == ch->rank) {
        out[(size_t)b * ch->world + q] = static_cast<char*>(mine[b]);
        continue;
      }
      if (r.buf_null[par][b]) continue;
      const std::string k = key_of(r.buf_h[par][b]);
      auto it = ch->opened.find(k);
      if (it == ch->opened.end()) {
        void* p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, r.buf_h[par][b], cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) MM_FAIL(MM_ECUDA, "ipc: open buffer %d of rank %d: %s", b, q, cudaGetErrorString(e));
        it = ch->opened.emplace(k, static_cast<char*>(p)).first;
      }
      out[(size_t)b * ch->world + q] = it->second + r.buf_off[par][b];
    }
  }
  return MM_OK;
}

mm_status ipc_allgather_u64(IpcChannel* ch, const uint64_t* row, int32_t n, std::vector<uint64_t>& out) {
  if (n > 64) MM_FAIL(MM_EINVAL, "ipc: row of %d", n);
  const int par = (int)(ch->rows++ & 1);
  std::memcpy(ch->shm->r[ch->rank].row[par], row, sizeof(uint64_t) * n);
  mm_status st = ipc_barrier(ch);
  if (st) return st;
  out.resize((size_t)n * ch->world);
  for (int32_t q = 0; q < ch->world; ++q) std::memcpy(&out[(size_t)q * n], ch->shm->r[q].row[par], sizeof(uint64_t) * n);
  return MM_OK;
}

}  // namespace mm
