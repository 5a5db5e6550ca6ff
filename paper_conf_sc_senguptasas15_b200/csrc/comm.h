// comm.h — the per-superstep exchange between owner partitions.
//
// Multi-GPU is the paper's future-work item (1) (§8). Destination
// intervals shard naturally: each rank owns a contiguous destination range, so
// one exchange per superstep suffices — an allgather of the changed vertices
// (frontier programs) or of the owned contribution slices (PageRank).
//   NcclComm : one process per GPU, NCCL over NVLink/NVSwitch (allgatherv as a
//              grouped ncclBroadcast from every root).
//   SimComm  : G "ranks" as host threads sharing ONE device (tests on a 1-GPU
//              box): the same protocol with device-to-device copies.
//   ShmComm  : one process per rank on one node (ranks may share a GPU): POSIX
//              shared memory for the host collectives, real cross-process
//              cudaIpc mappings for the device data (mailboxes, shared buffers).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "graphreduce.h"

namespace gr {

struct Comm {
  int rank = 0, world = 1;
  uint64_t bytes_in = 0;  // bytes received from peers (NVLink for NCCL)
  virtual ~Comm() = default;
  // allgatherv of device bytes: rank r's `counts[r]` bytes land at recv + displs[r]
  // on every rank. `send` may alias recv + displs[rank]. Stream-ordered on s.
  virtual gr_status allgatherv(const void *send, void *recv, const std::vector<uint64_t> &counts,
                               const std::vector<uint64_t> &displs, cudaStream_t s) = 0;
  // allgather of k host uint64 per rank (synchronous w.r.t. s): out[r*k + i]
  virtual gr_status allgather_small(const uint64_t *mine, int k, uint64_t *out, cudaStream_t s) = 0;
  // the same for k <= 8 uint64 already in DEVICE memory (stream-ordered after the
  // kernel that wrote them; one host synchronisation): out[r*k + i]
  virtual gr_status allgather_dev(const uint64_t *d_mine, int k, uint64_t *out, cudaStream_t s) = 0;
  // Map every rank's device buffer `local` into this rank: out[q] is rank q's
  // buffer (out[rank] = local). NCCL: cudaIpc handles exchanged with
  // allgather_small and opened with peer access (NVLink); the mappings are
  // closed when the Comm is destroyed. Simulated: the pointers themselves.
  // `local` must come from cudaMalloc (IPC-exportable). Collective: every rank
  // gets the same answer (GR_OK everywhere, or GR_EUNSUPPORTED everywhere when
  // some rank cannot export or map a peer buffer; the caller then falls back).
  virtual gr_status share_buffer(void *local, std::vector<void *> *out, cudaStream_t s) = 0;
  // Stream-ordered barrier: work enqueued on s after it starts only when every
  // rank's work enqueued before its barrier has completed (so peer stores of
  // those kernels are visible). NCCL: a one-word allreduce; simulated: host.
  virtual gr_status barrier(cudaStream_t s) = 0;
  // A rank that fails between collectives: make the peers' pending and next
  // collectives fail instead of waiting for it (NCCL: ncclCommAbort; shared
  // memory and simulated groups: the group is poisoned). The graph must be freed.
  virtual void abort_group() = 0;
  // Whether every rank runs in a CUDA context of its own (a process per rank). Kernels
  // that spin on a peer's stores (the device-side count exchange and barrier) need it:
  // streams of ONE context may share a hardware queue, so a spinning kernel could sit
  // in front of the very kernel it waits for (simulated ranks use the host paths).
  virtual bool own_context() const { return true; }
};

// Create the communicator for a loaded partition. world <= 1 returns nullptr.
// transport: kTransportNccl (one process per GPU), kTransportSim (in-process
// simulated group keyed by the 128-byte id), kTransportShm (one process per
// rank on one node, POSIX shared memory + cudaIpc; ranks may share a GPU).
constexpr int kTransportNccl = 0, kTransportShm = 1, kTransportSim = 2;
gr_status comm_create(int world, int rank, int transport, const void *id128, int device, Comm **out,
                      std::string *err);

}  // namespace gr
