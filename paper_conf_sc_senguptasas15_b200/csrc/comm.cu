// comm.cu — NCCL and simulated (in-process) partition exchange. See comm.h.
#include "comm.h"

#include <nccl.h>

#include <chrono>
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
    uint64_t *w = d_small + 8ull * world;
    return ncclAllReduce(w, w, 1, ncclUint64, ncclSum, comm, s) == ncclSuccess ? GR_OK : GR_ENCCL;
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
};

gr_status comm_create(int world, int rank, bool sim, const void *id128, int device, Comm **out, std::string *err) {
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
