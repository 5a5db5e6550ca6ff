// comm.cu — NCCL and simulated (in-process) partition exchange. See comm.h.
#include "comm.h"

#include <fcntl.h>
#include <nccl.h>
#include <sys/mman.h>
#include <unistd.h>

#include <atomic>
#include <chrono>
#include <thread>
#include <condition_variable>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>

namespace gr {

// ------------------------------------------------------------------- NCCL
struct NcclComm : Comm {
  ncclComm_t comm = nullptr;
  uint64_t *d_small = nullptr;  // world * 8 u64 scratch (+1 word for the barrier)
  uint64_t *h_small = nullptr;
  std::vector<void *> opened;   // cudaIpcOpenMemHandle mappings of peer buffers
  ~NcclComm() override {
    for (void *p : opened) cudaIpcCloseMemHandle(p);
    if (comm) ncclCommDestroy(comm);
    if (d_small) cudaFree(d_small);
    if (h_small) cudaFreeHost(h_small);
  }
  gr_status allgatherv(const void *send, void *recv, const std::vector<uint64_t> &counts,
                       const std::vector<uint64_t> &displs, cudaStream_t s) override {
    ncclResult_t r = ncclGroupStart();
    for (int q = 0; q < world && r == ncclSuccess; q++) {
      if (!counts[q]) continue;
      char *dst = static_cast<char *>(recv) + displs[q];
      r = ncclBroadcast(q == rank ? send : dst, dst, counts[q], ncclChar, q, comm, s);
      if (q != rank) bytes_in += counts[q];
    }
    ncclResult_t r2 = ncclGroupEnd();
    if (r != ncclSuccess || r2 != ncclSuccess) return GR_ENCCL;
    return GR_OK;
  }
  gr_status allgather_small(const uint64_t *mine, int k, uint64_t *out, cudaStream_t s) override {
    if (k > 8) return GR_EINVAL;
    if (cudaMemcpyAsync(d_small + (size_t)rank * 8, mine, 8 * k, cudaMemcpyHostToDevice, s) != cudaSuccess)
      return GR_ECUDA;
    if (ncclAllGather(d_small + (size_t)rank * 8, d_small, 8, ncclUint64, comm, s) != ncclSuccess) return GR_ENCCL;
    if (cudaMemcpyAsync(h_small, d_small, 64ull * world, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return GR_ECUDA;
    for (int q = 0; q < world; q++)
      for (int i = 0; i < k; i++) out[q * k + i] = h_small[q * 8 + i];
    return GR_OK;
  }
  gr_status allgather_dev(const uint64_t *d_mine, int k, uint64_t *out, cudaStream_t s) override {
    if (k > 8) return GR_EINVAL;
    if (ncclAllGather(d_mine, d_small, k, ncclUint64, comm, s) != ncclSuccess) return GR_ENCCL;
    if (cudaMemcpyAsync(h_small, d_small, 8ull * k * world, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return GR_ECUDA;
    for (int i = 0; i < k * world; i++) out[i] = h_small[i];
    return GR_OK;
  }
  // Every rank makes the same sequence of allgathers whatever happens locally, and
  // the result is agreed: GR_OK on all ranks or GR_EUNSUPPORTED on all ranks (a
  // rank without peer access must not leave the others waiting in a collective).
  gr_status share_buffer(void *local, std::vector<void *> *out, cudaStream_t s) override {
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle is 8 words");
    if (world > 64) return GR_EUNSUPPORTED;
    cudaIpcMemHandle_t h;
    std::memset(&h, 0, sizeof h);
    uint64_t ok = cudaIpcGetMemHandle(&h, local) == cudaSuccess ? 1 : 0;
    if (!ok) cudaGetLastError();
    uint64_t oks[64], mine[8], all[8 * 64];
    gr_status st = allgather_small(&ok, 1, oks, s);
    if (st != GR_OK) return st;
    for (int q = 0; q < world; q++)
      if (!oks[q]) return GR_EUNSUPPORTED;
    std::memcpy(mine, &h, 64);
    if ((st = allgather_small(mine, 8, all, s)) != GR_OK) return st;
    out->assign(world, nullptr);
    (*out)[rank] = local;
    std::vector<void *> mine_opened;
    ok = 1;
    for (int q = 0; q < world && ok; q++) {
      if (q == rank) continue;
      cudaIpcMemHandle_t hq;
      std::memcpy(&hq, all + 8 * q, 64);
      void *p = nullptr;
      if (cudaIpcOpenMemHandle(&p, hq, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        ok = 0;
        break;
      }
      mine_opened.push_back(p);
      (*out)[q] = p;
    }
    if ((st = allgather_small(&ok, 1, oks, s)) != GR_OK) return st;
    bool all_ok = true;
    for (int q = 0; q < world; q++) all_ok = all_ok && oks[q];
    if (!all_ok) {
      for (void *p : mine_opened) cudaIpcCloseMemHandle(p);
      out->clear();
      return GR_EUNSUPPORTED;
    }
    opened.insert(opened.end(), mine_opened.begin(), mine_opened.end());
    return GR_OK;
  }
  gr_status barrier(cudaStream_t s) override {
    if (!comm) return GR_ENCCL;
    uint64_t *w = d_small + 8ull * world;
    return ncclAllReduce(w, w, 1, ncclUint64, ncclSum, comm, s) == ncclSuccess ? GR_OK : GR_ENCCL;
  }
  void abort_group() override {
    if (comm) ncclCommAbort(comm);
    comm = nullptr;
  }
};

// -------------------------------------------------------------- simulated
struct SimGroup {
  int world = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  std::vector<const void *> ptrs;
  std::vector<uint64_t> small;  // world * 8
  int members = 0;
  bool poisoned = false;        // a rank failed: every waiter returns an error

  bool barrier() {
    std::unique_lock<std::mutex> lk(mu);
    if (poisoned) return false;
    const uint64_t g = gen;
    if (++arrived == world) {
      arrived = 0;
      gen++;
      cv.notify_all();
    } else {
      cv.wait_for(lk, std::chrono::seconds(300), [&] { return gen != g || poisoned; });
      if (gen == g) { poisoned = true; cv.notify_all(); return false; }
    }
    return !poisoned;
  }
  void poison() {
    std::lock_guard<std::mutex> lk(mu);
    poisoned = true;
    cv.notify_all();
  }
};

static std::mutex g_sim_mu;
static std::map<std::string, std::shared_ptr<SimGroup>> g_sim_groups;

struct SimComm : Comm {
  std::shared_ptr<SimGroup> grp;
  std::string key;
  ~SimComm() override {
    std::lock_guard<std::mutex> lk(g_sim_mu);
    if (--grp->members == 0) g_sim_groups.erase(key);
  }
  gr_status fail_all(gr_status s) {
    grp->poison();
    return s;
  }
  gr_status allgatherv(const void *send, void *recv, const std::vector<uint64_t> &counts,
                       const std::vector<uint64_t> &displs, cudaStream_t s) override {
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);  // own data ready
    grp->ptrs[rank] = send;
    if (!grp->barrier()) return GR_ENCCL;
    for (int q = 0; q < world; q++) {
      char *dst = static_cast<char *>(recv) + displs[q];
      if (!counts[q] || grp->ptrs[q] == dst) continue;
      if (cudaMemcpyAsync(dst, grp->ptrs[q], counts[q], cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        return fail_all(GR_ECUDA);
      if (q != rank) bytes_in += counts[q];
    }
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    if (!grp->barrier()) return GR_ENCCL;  // peers may reuse their send buffers only after everyone copied
    return GR_OK;
  }
  gr_status allgather_small(const uint64_t *mine, int k, uint64_t *out, cudaStream_t s) override {
    if (k > 8) return fail_all(GR_EINVAL);
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    for (int i = 0; i < k; i++) grp->small[rank * 8 + i] = mine[i];
    if (!grp->barrier()) return GR_ENCCL;
    for (int q = 0; q < world; q++)
      for (int i = 0; i < k; i++) out[q * k + i] = grp->small[q * 8 + i];
    if (!grp->barrier()) return GR_ENCCL;
    return GR_OK;
  }
  gr_status allgather_dev(const uint64_t *d_mine, int k, uint64_t *out, cudaStream_t s) override {
    if (k > 8) return fail_all(GR_EINVAL);
    uint64_t mine[8];
    if (cudaMemcpyAsync(mine, d_mine, 8ull * k, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return fail_all(GR_ECUDA);
    return allgather_small(mine, k, out, s);
  }
  gr_status share_buffer(void *local, std::vector<void *> *out, cudaStream_t s) override {
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    grp->ptrs[rank] = local;
    if (!grp->barrier()) return GR_ENCCL;
    out->resize(world);
    for (int q = 0; q < world; q++) (*out)[q] = const_cast<void *>(grp->ptrs[q]);
    if (!grp->barrier()) return GR_ENCCL;  // ptrs is reused by the next exchange
    return GR_OK;
  }
  gr_status barrier(cudaStream_t s) override {
    // ranks share one device: wait for this rank's work, then for every rank's
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    return grp->barrier() ? GR_OK : GR_ENCCL;
  }
  void abort_group() override { grp->poison(); }
  bool own_context() const override { return false; }  // threads of one process share a context
};

// ------------------------------------------------- process-shared memory
// One process per rank on ONE node, ranks possibly sharing a GPU (NCCL refuses
// two ranks on one device): host-side collectives through a POSIX shared-memory
// segment named after the 128-byte id, device data through real cross-process
// cudaIpc mappings — every rank's mailbox (allgatherv) and every buffer handed
// to share_buffer (the fused PageRank / frontier exchanges store into them
// from the kernels). This is the same protocol the NCCL communicator runs,
// with the IPC path taken for real between processes.
struct ShmHdr {
  std::atomic<uint64_t> arrived, gen;
  std::atomic<uint32_t> poisoned, attached;
  uint64_t small[64 * 8];    // allgather_small slots
};
static_assert(std::atomic<uint64_t>::is_always_lock_free, "cross-process atomics");

struct ShmComm : Comm {
  ShmHdr *h = nullptr;
  std::string name;
  void *mbox = nullptr;            // this rank's device mailbox (cudaMalloc, IPC-exported)
  uint64_t mbox_cap = 0;
  std::vector<void *> peer_mbox;   // mapped mailboxes of every rank (own included)
  std::vector<void *> opened;      // every cudaIpcOpenMemHandle mapping, closed at destruction
  ~ShmComm() override {
    for (void *p : opened) cudaIpcCloseMemHandle(p);
    if (mbox) cudaFree(mbox);
    if (h) {
      const bool last = h->attached.fetch_sub(1) == 1;
      munmap(h, sizeof(ShmHdr));
      if (last) shm_unlink(name.c_str());
    }
  }
  bool host_barrier() {
    if (h->poisoned.load()) return false;
    const uint64_t g = h->gen.load();
    if (h->arrived.fetch_add(1) + 1 == (uint64_t)world) {
      h->arrived.store(0);
      h->gen.fetch_add(1);
      return true;
    }
    const auto t0 = std::chrono::steady_clock::now();
    for (uint64_t spins = 0; h->gen.load() == g; spins++) {
      if (h->poisoned.load()) return false;
      if (spins > 1000) std::this_thread::sleep_for(std::chrono::microseconds(20));
      if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(300)) {
        h->poisoned.store(1);
        return false;
      }
    }
    return !h->poisoned.load();
  }
  gr_status fail_all(gr_status s) {
    h->poisoned.store(1);
    return s;
  }
  gr_status allgather_small(const uint64_t *mine, int k, uint64_t *out, cudaStream_t s) override {
    if (k > 8) return fail_all(GR_EINVAL);
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    for (int i = 0; i < k; i++) h->small[rank * 8 + i] = mine[i];
    if (!host_barrier()) return GR_ENCCL;
    for (int q = 0; q < world; q++)
      for (int i = 0; i < k; i++) out[q * k + i] = h->small[q * 8 + i];
    if (!host_barrier()) return GR_ENCCL;
    return GR_OK;
  }
  gr_status allgather_dev(const uint64_t *d_mine, int k, uint64_t *out, cudaStream_t s) override {
    if (k > 8) return fail_all(GR_EINVAL);
    uint64_t mine[8];
    if (cudaMemcpyAsync(mine, d_mine, 8ull * k, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return fail_all(GR_ECUDA);
    return allgather_small(mine, k, out, s);
  }
  // export `local` (cudaMalloc) and open every peer's export; agreed on every rank
  gr_status exchange_handles(void *local, std::vector<void *> *out, cudaStream_t s) {
    cudaIpcMemHandle_t hd;
    std::memset(&hd, 0, sizeof hd);
    uint64_t ok = cudaIpcGetMemHandle(&hd, local) == cudaSuccess ? 1 : 0;
    if (!ok) cudaGetLastError();
    uint64_t oks[64], mine[8], all[8 * 64];
    gr_status st = allgather_small(&ok, 1, oks, s);
    if (st != GR_OK) return st;
    for (int q = 0; q < world; q++)
      if (!oks[q]) return GR_EUNSUPPORTED;
    std::memcpy(mine, &hd, 64);
    if ((st = allgather_small(mine, 8, all, s)) != GR_OK) return st;
    out->assign(world, nullptr);
    (*out)[rank] = local;
    std::vector<void *> mine_opened;
    ok = 1;
    for (int q = 0; q < world && ok; q++) {
      if (q == rank) continue;
      cudaIpcMemHandle_t hq;
      std::memcpy(&hq, all + 8 * q, 64);
      void *p = nullptr;
      if (cudaIpcOpenMemHandle(&p, hq, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        ok = 0;
        break;
      }
      mine_opened.push_back(p);
      (*out)[q] = p;
    }
    if ((st = allgather_small(&ok, 1, oks, s)) != GR_OK) return st;
    bool all_ok = true;
    for (int q = 0; q < world; q++) all_ok = all_ok && oks[q];
    if (!all_ok) {
      for (void *p : mine_opened) cudaIpcCloseMemHandle(p);
      out->clear();
      return GR_EUNSUPPORTED;
    }
    opened.insert(opened.end(), mine_opened.begin(), mine_opened.end());
    return GR_OK;
  }
  gr_status share_buffer(void *local, std::vector<void *> *out, cudaStream_t s) override {
    if (world > 64) return GR_EUNSUPPORTED;
    return exchange_handles(local, out, s);
  }
  // Every rank copies its slice into its own mailbox, then (after a barrier) reads
  // every peer's slice from the peer's mapped mailbox; mailboxes grow in lockstep
  // (every rank knows every count, so all agree on the capacity).
  gr_status allgatherv(const void *send, void *recv, const std::vector<uint64_t> &counts,
                       const std::vector<uint64_t> &displs, cudaStream_t s) override {
    uint64_t need = 0;
    for (int q = 0; q < world; q++) need = counts[q] > need ? counts[q] : need;
    if (need > mbox_cap) {
      uint64_t cap = mbox_cap ? mbox_cap : (1u << 20);
      while (cap < need) cap *= 2;
      if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
      if (!host_barrier()) return GR_ENCCL;  // nobody reads the old mailboxes any more
      for (int q = 0; q < world; q++)
        if (q != rank && peer_mbox.size() == (size_t)world && peer_mbox[q]) {
          cudaIpcCloseMemHandle(peer_mbox[q]);
          for (auto it = opened.begin(); it != opened.end(); ++it)
            if (*it == peer_mbox[q]) { opened.erase(it); break; }
        }
      if (mbox) cudaFree(mbox);
      mbox = nullptr;
      mbox_cap = 0;
      if (cudaMalloc(&mbox, cap) != cudaSuccess) {
        cudaGetLastError();
        return fail_all(GR_ENOMEM);
      }
      mbox_cap = cap;
      gr_status st = exchange_handles(mbox, &peer_mbox, s);
      if (st != GR_OK) return fail_all(st == GR_EUNSUPPORTED ? GR_ECUDA : st);
    }
    if (counts[rank] &&
        cudaMemcpyAsync(mbox, send, counts[rank], cudaMemcpyDeviceToDevice, s) != cudaSuccess)
      return fail_all(GR_ECUDA);
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    if (!host_barrier()) return GR_ENCCL;
    for (int q = 0; q < world; q++) {
      char *dst = static_cast<char *>(recv) + displs[q];
      if (!counts[q] || (q == rank && send == dst)) continue;
      if (cudaMemcpyAsync(dst, q == rank ? send : peer_mbox[q], counts[q], cudaMemcpyDeviceToDevice, s) !=
          cudaSuccess)
        return fail_all(GR_ECUDA);
      if (q != rank) bytes_in += counts[q];
    }
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    if (!host_barrier()) return GR_ENCCL;  // mailboxes may be rewritten only after everyone copied
    return GR_OK;
  }
  gr_status barrier(cudaStream_t s) override {
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail_all(GR_ECUDA);
    return host_barrier() ? GR_OK : GR_ENCCL;
  }
  void abort_group() override { h->poisoned.store(1); }
};

static gr_status shm_create(int world, int rank, const void *id128, ShmComm **out, std::string *err) {
  static const char hex[] = "0123456789abcdef";
  std::string name = "/gr_shm_";
  const unsigned char *b = static_cast<const unsigned char *>(id128);
  for (int i = 0; i < 16; i++) {
    name += hex[b[i] >> 4];
    name += hex[b[i] & 15];
  }
  const int fd = shm_open(name.c_str(), O_CREAT | O_RDWR, 0600);
  if (fd < 0) {
    *err = "shm_open " + name + " failed";
    return GR_EINVAL;
  }
  if (ftruncate(fd, sizeof(ShmHdr)) != 0) {  // every rank: the same size (zero-filled once)
    close(fd);
    *err = "ftruncate of the shared segment failed";
    return GR_ENOMEM;
  }
  void *p = mmap(nullptr, sizeof(ShmHdr), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (p == MAP_FAILED) {
    *err = "mmap of the shared segment failed";
    return GR_ENOMEM;
  }
  auto *c = new ShmComm();
  c->rank = rank;
  c->world = world;
  c->name = name;
  c->h = static_cast<ShmHdr *>(p);
  c->h->attached.fetch_add(1);
  *out = c;
  return GR_OK;
}

gr_status comm_create(int world, int rank, int transport, const void *id128, int device, Comm **out,
                      std::string *err) {
  if (transport == kTransportShm) {
    *out = nullptr;
    if (world <= 1) return GR_OK;
    if (!id128) {
      *err = "world > 1 needs a 128-byte group id";
      return GR_EINVAL;
    }
    if (world > 64) {
      *err = "shared-memory transport: world <= 64";
      return GR_EINVAL;
    }
    cudaSetDevice(device);
    ShmComm *c = nullptr;
    gr_status st = shm_create(world, rank, id128, &c, err);
    if (st != GR_OK) return st;
    // every rank attached and alive before the first collective
    if (!c->host_barrier()) {
      delete c;
      *err = "shared-memory group: ranks did not all attach within 300 s";
      return GR_ENCCL;
    }
    *out = c;
    return GR_OK;
  }
  const bool sim = transport == kTransportSim;
  *out = nullptr;
  if (world <= 1) return GR_OK;
  if (!id128) {
    *err = "world > 1 needs nccl_unique_id (128 bytes; any 128 bytes name a simulated group)";
    return GR_EINVAL;
  }
  if (sim) {
    auto *c = new SimComm();
    c->rank = rank;
    c->world = world;
    c->key.assign(static_cast<const char *>(id128), 128);
    {
      std::lock_guard<std::mutex> lk(g_sim_mu);
      auto &g = g_sim_groups[c->key];
      if (!g) {
        g = std::make_shared<SimGroup>();
        g->world = world;
        g->ptrs.assign(world, nullptr);
        g->small.assign(8ull * world, 0);
      }
      g->members++;
      c->grp = g;
      if (g->world != world) {
        delete c;
        *err = "simulated group world mismatch";
        return GR_EINVAL;
      }
    }
    *out = c;
    return GR_OK;
  }
  auto *c = new NcclComm();
  c->rank = rank;
  c->world = world;
  ncclUniqueId id;
  std::memcpy(&id, id128, sizeof id);
  cudaSetDevice(device);
  ncclResult_t r = ncclCommInitRank(&c->comm, world, id, rank);
  if (r != ncclSuccess) {
    *err = std::string("ncclCommInitRank: ") + ncclGetErrorString(r);
    c->comm = nullptr;
    delete c;
    return GR_ENCCL;
  }
  if (cudaMalloc(&c->d_small, 64ull * world + 64) != cudaSuccess ||
      cudaMallocHost(&c->h_small, 64ull * world) != cudaSuccess) {
    delete c;
    *err = "comm scratch allocation failed";
    return GR_ENOMEM;
  }
  *out = c;
  return GR_OK;
}

}  // namespace gr
