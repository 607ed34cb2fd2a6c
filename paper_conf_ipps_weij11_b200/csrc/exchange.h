// Multi-GPU exchange transports: one rank per GPU, each rank owns the trie
// collections b with b mod K == rank.  Two collectives are needed per chunk: an
// all-gather of a few u64 counts and an all-to-all-v of byte buffers.
//   * NcclTransport: NCCL 2.28 (loaded with dlopen, so single-GPU use never needs libnccl);
//     all-to-all-v = ncclGroupStart + per-peer ncclSend/ncclRecv on the context stream (NVLink 5 /
//     NVSwitch on a B200 box).
//   * LoopbackTransport: K contexts of one process (one host thread each) sharing a hub; the same
//     pack/unpack code runs, the bytes move with device-to-device cudaMemcpyAsync.  Used to test the
//     protocol on a single GPU.
#pragma once
#include <dlfcn.h>

#include <condition_variable>
#include <cstdint>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include <cuda_runtime.h>
#include <nccl.h>

namespace wj {

struct ExchangeError {
  std::string msg;
};

struct Transport {
  int rank = 0, world = 1;
  uint64_t sent = 0;  // bytes sent to other ranks
  virtual ~Transport() {}
  // all[r*n + i] = value i of rank r (host buffers)
  virtual void allgather(const uint64_t* mine, size_t n, uint64_t* all, cudaStream_t st) = 0;
  // device byte buffers; soff/roff: K+1 host byte offsets (segment p goes to / comes from rank p)
  virtual void alltoallv(const void* send, const uint64_t* soff, void* recv, const uint64_t* roff, cudaStream_t st) = 0;
};

// ------------------------------------------------------------------ loopback
struct LoopbackHub {
  int world;
  std::mutex m;
  std::condition_variable cv;
  int count = 0;
  uint64_t gen = 0;
  std::vector<std::vector<uint64_t>> vals;
  std::vector<const void*> ptrs;
  std::vector<std::vector<uint64_t>> offs;
  explicit LoopbackHub(int w) : world(w), vals(w), ptrs(w), offs(w) {}
  void barrier() {
    std::unique_lock<std::mutex> lk(m);
    const uint64_t g = gen;
    if (++count == world) {
      count = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g; });
    }
  }
};

struct LoopbackTransport : Transport {
  LoopbackHub* hub;
  LoopbackTransport(LoopbackHub* h, int r) : hub(h) {
    rank = r;
    world = h->world;
  }
  void allgather(const uint64_t* mine, size_t n, uint64_t* all, cudaStream_t) override {
    hub->vals[rank].assign(mine, mine + n);
    hub->barrier();
    for (int r = 0; r < world; ++r) memcpy(all + (size_t)r * n, hub->vals[r].data(), n * 8);
    hub->barrier();
  }
  void alltoallv(const void* send, const uint64_t* soff, void* recv, const uint64_t* roff, cudaStream_t st) override {
    if (cudaStreamSynchronize(st) != cudaSuccess) throw ExchangeError{"loopback: stream sync failed"};
    hub->ptrs[rank] = send;
    hub->offs[rank].assign(soff, soff + world + 1);
    hub->barrier();
    for (int s = 0; s < world; ++s) {
      const uint64_t a = hub->offs[s][rank], b = hub->offs[s][rank + 1];
      if (b - a != roff[s + 1] - roff[s]) throw ExchangeError{"loopback: size mismatch"};
      if (b > a &&
          cudaMemcpyAsync((char*)recv + roff[s], (const char*)hub->ptrs[s] + a, b - a, cudaMemcpyDeviceToDevice, st) !=
              cudaSuccess)
        throw ExchangeError{"loopback: copy failed"};
    }
    if (cudaStreamSynchronize(st) != cudaSuccess) throw ExchangeError{"loopback: copy sync failed"};
    hub->barrier();
    sent += soff[world] - (soff[rank + 1] - soff[rank]);
  }

};

// ------------------------------------------------------------------ NCCL (dlopen)
struct NcclApi {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;

  static NcclApi& get() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
      const char* env = getenv("WJ_NCCL_LIB");
      const char* names[] = {env, "libnccl.so.2", "libnccl.so"};
      for (const char* n : names) {
        if (!n) continue;
        api.h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
        if (api.h) break;
      }
      if (!api.h) return;
#define WJ_SYM(f) api.f = (decltype(api.f))dlsym(api.h, "nccl" #f)
      WJ_SYM(GetUniqueId); WJ_SYM(CommInitRank); WJ_SYM(CommDestroy); WJ_SYM(AllGather); WJ_SYM(Send);
      WJ_SYM(Recv); WJ_SYM(GroupStart); WJ_SYM(GroupEnd); WJ_SYM(GetErrorString);
#undef WJ_SYM
    });
    if (!api.h || !api.CommInitRank || !api.Send) throw ExchangeError{"libnccl.so.2 not found (set WJ_NCCL_LIB)"};
    return api;
  }
};

inline void nccl_check(ncclResult_t r, const char* what) {
  if (r != ncclSuccess) {
    NcclApi& a = NcclApi::get();
    throw ExchangeError{std::string(what) + ": " + (a.GetErrorString ? a.GetErrorString(r) : "nccl error")};
  }
}

struct NcclTransport : Transport {
  ncclComm_t comm = nullptr;
  uint64_t* dbuf = nullptr;  // device scratch for all-gathers
  size_t dcap = 0;
  NcclTransport(const void* uid, int r, int w) {
    rank = r;
    world = w;
    NcclApi& a = NcclApi::get();
    ncclUniqueId id;
    memcpy(&id, uid, sizeof(id));
    nccl_check(a.CommInitRank(&comm, w, id, r), "ncclCommInitRank");
  }
  ~NcclTransport() override {
    if (dbuf) cudaFree(dbuf);
    if (comm) NcclApi::get().CommDestroy(comm);
  }
  void allgather(const uint64_t* mine, size_t n, uint64_t* all, cudaStream_t st) override {
    const size_t need = n * (world + 1);
    if (need > dcap) {
      if (dbuf) cudaFree(dbuf);
      if (cudaMalloc(&dbuf, need * 8) != cudaSuccess) throw ExchangeError{"allgather scratch alloc"};
      dcap = need;
    }
    if (cudaMemcpyAsync(dbuf, mine, n * 8, cudaMemcpyHostToDevice, st) != cudaSuccess) throw ExchangeError{"h2d"};
    nccl_check(NcclApi::get().AllGather(dbuf, dbuf + n, n, ncclUint64, comm, st), "ncclAllGather");
    if (cudaMemcpyAsync(all, dbuf + n, n * world * 8, cudaMemcpyDeviceToHost, st) != cudaSuccess) throw ExchangeError{"d2h"};
    if (cudaStreamSynchronize(st) != cudaSuccess) throw ExchangeError{"allgather sync"};
  }
  void alltoallv(const void* send, const uint64_t* soff, void* recv, const uint64_t* roff, cudaStream_t st) override {
    NcclApi& a = NcclApi::get();
    // the rank's own segment never leaves the GPU: a device copy, not an NCCL self send/recv
    const uint64_t own = soff[rank + 1] - soff[rank];
    if (own != roff[rank + 1] - roff[rank]) throw ExchangeError{"alltoallv: self size mismatch"};
    if (own && cudaMemcpyAsync((char*)recv + roff[rank], (const char*)send + soff[rank], own, cudaMemcpyDeviceToDevice,
                               st) != cudaSuccess)
      throw ExchangeError{"alltoallv: self copy failed"};
    nccl_check(a.GroupStart(), "ncclGroupStart");
    for (int p = 0; p < world; ++p) {
      if (p == rank) continue;
      const uint64_t sb = soff[p + 1] - soff[p], rb = roff[p + 1] - roff[p];
      if (sb) nccl_check(a.Send((const char*)send + soff[p], sb, ncclChar, p, comm, st), "ncclSend");
      if (rb) nccl_check(a.Recv((char*)recv + roff[p], rb, ncclChar, p, comm, st), "ncclRecv");
    }
    nccl_check(a.GroupEnd(), "ncclGroupEnd");
    sent += soff[world] - (soff[rank + 1] - soff[rank]);
  }

};

// ------------------------------------------------------------------ K-way merge of serialized slices
// Each rank's index_serialize output holds the terms of the collections it owns (disjoint, sorted);
// the global inverted file is their merge by term bytes (host, untimed).  Header counts add up except
// n_docs (global in every slice).
struct SliceView {
  const uint8_t* base;
  bool vb;  // WJINV002: post_off in bytes into `code` (reading S19)
  uint64_t n_docs, n_tokens, n_dropped, n_terms, n_postings, n_tb, n_pb;
  const uint64_t* term_off;
  const uint8_t* term_bytes;
  const uint32_t* df;
  const uint64_t* cf;
  const uint64_t* post_off;
  const uint32_t* docid;
  const uint32_t* tf;
  const uint8_t* code;
};

inline uint64_t pad8(uint64_t x) { return (x + 7) & ~7ull; }

inline bool parse_slice(const uint8_t* b, uint64_t size, SliceView& v) {
  if (size < 64) return false;
  v.vb = memcmp(b, "WJINV002", 8) == 0;
  if (!v.vb && memcmp(b, "WJINV001", 8) != 0) return false;
  const uint64_t* h = (const uint64_t*)b;
  v.base = b;
  v.n_docs = h[1]; v.n_tokens = h[2]; v.n_dropped = h[3]; v.n_terms = h[4]; v.n_postings = h[5]; v.n_tb = h[6];
  v.n_pb = v.vb ? h[7] : 0;
  uint64_t p = 64;
  v.term_off = (const uint64_t*)(b + p); p += 8 * (v.n_terms + 1);
  v.term_bytes = b + p; p += pad8(v.n_tb);
  v.df = (const uint32_t*)(b + p); p += pad8(4 * v.n_terms);
  v.cf = (const uint64_t*)(b + p); p += 8 * v.n_terms;
  v.post_off = (const uint64_t*)(b + p); p += 8 * (v.n_terms + 1);
  v.docid = v.tf = nullptr;
  v.code = nullptr;
  if (v.vb) {
    v.code = b + p; p += pad8(v.n_pb);
  } else {
    v.docid = (const uint32_t*)(b + p); p += pad8(4 * v.n_postings);
    v.tf = (const uint32_t*)(b + p); p += pad8(4 * v.n_postings);
  }
  return p == size;
}

}  // namespace wj
