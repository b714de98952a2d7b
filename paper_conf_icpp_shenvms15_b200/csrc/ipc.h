// Multi-process transport of the executor (world > 1, one logical device per
// process, all processes on one node): a POSIX shared-memory rendezvous block
// for the host-side control plane (IPC handles, a host barrier, profile rows)
// and device-memory completion flags that ranks signal and wait on through
// CUDA IPC mappings.  Data moves as pulls: a consumer copies the elements it
// needs straight out of the producer's buffer (peer memory over NVLink on a
// multi-GPU node, the same HBM when ranks share a GPU), so the op program's
// exact hazards (RAW on the producer, WAR on the reader) become flag waits.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <map>
#include <string>
#include <vector>

#include "mm.h"

namespace mm {

constexpr int64_t kIpcFlagSlots = 1 << 20;   // uint64 flags per rank (8 MiB)
constexpr int64_t kIpcEpoch = 0;             // flags[0]: this rank's run counter
constexpr int64_t kIpcEnd = 1;               // flags[1]: run epoch whose every op is done
constexpr int64_t kIpcOp0 = 8;               // flags[8 + i]: op i of the current program

struct ShmRank {
  uint64_t pid;
  cudaIpcMemHandle_t flags_h;
  // buffer table, double-buffered by run parity
  int32_t nbuf[2];
  cudaIpcMemHandle_t buf_h[2][MM_MAX_BUF];
  uint64_t buf_off[2][MM_MAX_BUF];
  uint64_t buf_null[2][MM_MAX_BUF];
  uint64_t row[2][64];                       // small per-rank exchange rows (profile, tuning)
};

struct ShmBlock {
  uint32_t magic;
  int32_t world;
  int32_t attached;
  uint32_t bar_count;
  uint32_t bar_gen;
  int32_t failed;
  ShmRank r[MM_MAX_DEV];
};

struct IpcChannel {
  int32_t world = 1, rank = 0;
  ShmBlock* shm = nullptr;
  std::string name;
  uint64_t* flags = nullptr;                 // this rank's flags (device)
  std::vector<uint64_t*> peer_flags;         // per rank, mapped (own = flags)
  std::map<std::string, char*> opened;       // handle bytes -> mapped base (peers)
  std::map<const void*, std::pair<cudaIpcMemHandle_t, uint64_t>> exported;  // ptr -> (handle, offset)
  uint64_t xchg = 0;                         // buffer-table exchanges done
  uint64_t rows = 0;                         // row exchanges done
};

// Create / attach the rendezvous block named after the 128-byte id, allocate
// this rank's flags on the current device, exchange the flag handles.
mm_status ipc_open(IpcChannel* ch, const void* id128, int32_t rank, int32_t world);
void ipc_close(IpcChannel* ch);
// Host barrier over all ranks (spins on shared memory; fails after a timeout).
mm_status ipc_barrier(IpcChannel* ch);
// Publish this rank's pointers of every buffer slot and map every peer's:
// out[slot * world + rank] = a pointer valid in this process (own pointer for
// this rank, the IPC mapping for peers, NULL where a rank has none).
mm_status ipc_exchange_buffers(IpcChannel* ch, const std::vector<void*>& mine, std::vector<char*>& out);
// All-gather `n` <= 64 uint64 per rank: out[r * n + i].
mm_status ipc_allgather_u64(IpcChannel* ch, const uint64_t* row, int32_t n, std::vector<uint64_t>& out);

// Device side (stream-ordered, CUDA-graph capturable).
cudaError_t ipc_bump_epoch(uint64_t* flags, cudaStream_t s);
cudaError_t ipc_signal(uint64_t* flags, int64_t slot, cudaStream_t s);
// Wait until every peer_flags[i][slot[i]] >= this rank's epoch - lag[i].
cudaError_t ipc_wait(const uint64_t* my_flags, uint64_t* const* peer, const int64_t* slot, const uint32_t* lag,
                     int32_t n, cudaStream_t s);

}  // namespace mm
