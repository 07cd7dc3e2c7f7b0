// Host runtime behind include/msccl.h: communicators, shared regions, program loading,
// program selection by size range (MSCCLang §6), geometry, launch.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <sstream>
#include <string>
#include <tuple>
#include <vector>

#include "../../include/msccl.h"
#include "device.h"
#include "ir.h"
#include "kernels.h"

using namespace msccl;

// ------------------------------------------------------------------ parameters
namespace {

struct Params {
  int64_t slots = 4, slotBytes = 262144, maxChannels = 32, threads = 512, timeoutS = 20, tma = 0, direct = 1,
          warp = 0, l2PersistMiB = 0, prefetch = 0, directTile = 1, balance = 0, directHints = 1;
};

std::mutex gMu;
Params gParams;
bool gEnvRead = false;
std::string gLastError;
std::atomic<uint64_t> gLaunches{0};

int64_t* paramRef(Params& p, const std::string& k) {
  if (k == "MSCCL_SLOTS") return &p.slots;
  if (k == "MSCCL_SLOT_BYTES") return &p.slotBytes;
  if (k == "MSCCL_MAX_CHANNELS") return &p.maxChannels;
  if (k == "MSCCL_THREADS") return &p.threads;
  if (k == "MSCCL_TIMEOUT_S") return &p.timeoutS;
  if (k == "MSCCL_TMA") return &p.tma;
  if (k == "MSCCL_DIRECT") return &p.direct;
  if (k == "MSCCL_WARP_FLAGS") return &p.warp;
  if (k == "MSCCL_L2_PERSIST_MIB") return &p.l2PersistMiB;
  if (k == "MSCCL_PREFETCH") return &p.prefetch;
  if (k == "MSCCL_DIRECT_TILE") return &p.directTile;
  if (k == "MSCCL_BALANCE") return &p.balance;
  if (k == "MSCCL_DIRECT_HINTS") return &p.directHints;
  return nullptr;
}

Params currentParams() {
  std::lock_guard<std::mutex> g(gMu);
  if (!gEnvRead) {
    gEnvRead = true;
    for (const char* k : {"MSCCL_SLOTS", "MSCCL_SLOT_BYTES", "MSCCL_MAX_CHANNELS", "MSCCL_THREADS", "MSCCL_TIMEOUT_S",
                          "MSCCL_TMA", "MSCCL_DIRECT", "MSCCL_WARP_FLAGS",
                          "MSCCL_L2_PERSIST_MIB", "MSCCL_PREFETCH", "MSCCL_DIRECT_TILE",
                          "MSCCL_BALANCE", "MSCCL_DIRECT_HINTS"}) {
      const char* v = getenv(k);
      if (v && *v) *paramRef(gParams, k) = atoll(v);
    }
  }
  return gParams;
}

int elemBytes(int dt) {
  static const int w[10] = {1, 1, 4, 4, 8, 8, 2, 4, 8, 2};
  return (dt >= 0 && dt < 10) ? w[dt] : 0;
}

bool debugOn() {
  const char* v = getenv("MSCCL_DEBUG");
  return v && (strcmp(v, "INFO") == 0 || strcmp(v, "1") == 0);
}

}  // namespace

// ------------------------------------------------------------------ objects
struct Clique {  // ranks created together by mscclCommInitAll
  std::vector<mscclComm*> comms;
};

struct mscclProgram;

struct mscclComm {
  int nranks = 0, rank = 0, dev = 0;
  Params prm;
  // shared region (receiver-side FIFOs + flags), one cudaMalloc so it can be IPC-exported
  char* region = nullptr;
  size_t regionBytes = 0, fifoBytes = 0, flagsOff = 0;
  std::vector<char*> peerBase;
  std::vector<bool> peerIpc;
  bool connected = false;
  bool sysScope = false;
  uint32_t* hostAbort = nullptr;     // pinned, mapped
  uint32_t* hostAbortDev = nullptr;  // device alias
  std::shared_ptr<Clique> clique;
  std::vector<mscclProgram*> programs;
  std::string lastError;
  int maxCoResident = 0;

  // region layout
  size_t fifoOff(int src, int ch) const {
    return ((size_t)src * prm.maxChannels + ch) * prm.slots * prm.slotBytes;
  }
  // kind: 0 head, 1 ack, 2 sendCnt, 3 recvCnt; MSCCL_FLAG_WORDS words (one 128-byte line) each
  size_t flagOff(int kind, int peer, int ch) const {
    return flagsOff + (((size_t)kind * nranks + peer) * prm.maxChannels + ch) * MSCCL_FLAG_WORDS * sizeof(uint64_t);
  }
  size_t abortOff() const { return flagOff(4, 0, 0); }
};

struct mscclProgram {
  mscclComm* comm = nullptr;
  Algo algo;
  size_t minBytes = 0, maxBytes = 0;
  int index = 0;
  int nTB = 0, nInstr = 0;
  DevTB* dTBs = nullptr;
  DevInstr* dInstr = nullptr;
  uint64_t* dDeps = nullptr;
  uint64_t* dSem = nullptr;  // nTB sems followed by nTB gens
  char* dScratch = nullptr;
  size_t scratchBytes = 0;
  int maxCnt = 1;
  bool hasReduce = false;
  bool allDirect = true;  // every message of this rank's program is a direct placement (R15)
  std::vector<int64_t> tbWork;        // chunk-sized operand touches per thread block (FIFO protocol)
  std::vector<int64_t> tbWorkDirect;  // ... with direct placement (R15)
};

namespace {

mscclResult_t setErr(mscclComm* c, mscclResult_t r, const std::string& msg) {
  std::lock_guard<std::mutex> g(gMu);
  gLastError = msg;
  if (c) c->lastError = msg;
  if (debugOn()) fprintf(stderr, "[msccl] error %d: %s\n", (int)r, msg.c_str());
  return r;
}

#define CUDACHECK(c, call)                                                                          \
  do {                                                                                              \
    cudaError_t e_ = (call);                                                                        \
    if (e_ != cudaSuccess) {                                                                        \
      return setErr((c), mscclUnhandledCudaError,                                                   \
                    std::string(#call) + ": " + cudaGetErrorString(e_));                           \
    }                                                                                               \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) {
    cudaGetDevice(&prev);
    if (prev != d) cudaSetDevice(d);
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

mscclResult_t allocRegion(mscclComm* c) {
  c->prm = currentParams();
  if (c->prm.slots < 1 || c->prm.slots > 16) return setErr(c, mscclInvalidArgument, "MSCCL_SLOTS must be in 1..16");
  if (c->prm.slotBytes < 4096 || c->prm.slotBytes % 256) return setErr(c, mscclInvalidArgument, "MSCCL_SLOT_BYTES must be a multiple of 256, >= 4096");
  if (c->prm.threads < 64 || c->prm.threads > 512 || c->prm.threads % 32) return setErr(c, mscclInvalidArgument, "MSCCL_THREADS must be a multiple of 32 in 64..512");
  if (c->prm.maxChannels < 1 || c->prm.maxChannels > 1024) return setErr(c, mscclInvalidArgument, "MSCCL_MAX_CHANNELS out of range");
  DeviceGuard g(c->dev);
  c->fifoBytes = (size_t)c->nranks * c->prm.maxChannels * c->prm.slots * c->prm.slotBytes;
  c->flagsOff = c->fifoBytes;
  c->regionBytes = c->abortOff() + 256;
  CUDACHECK(c, cudaMalloc(&c->region, c->regionBytes));
  CUDACHECK(c, cudaMemset(c->region, 0, c->regionBytes));
  // optional L2 set-aside for evict_last (persisting) lines: the FIFO slot stores carry
  // L2::evict_last, which only has a reserved home when the set-aside is non-zero
  if (c->prm.l2PersistMiB > 0)
    CUDACHECK(c, cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)c->prm.l2PersistMiB << 20));
  CUDACHECK(c, cudaHostAlloc(&c->hostAbort, sizeof(uint32_t), cudaHostAllocMapped | cudaHostAllocPortable));
  *c->hostAbort = 0;
  CUDACHECK(c, cudaHostGetDevicePointer((void**)&c->hostAbortDev, c->hostAbort, 0));
  c->peerBase.assign(c->nranks, nullptr);
  c->peerIpc.assign(c->nranks, false);
  c->peerBase[c->rank] = c->region;
  int nsm = 0, nb = 0;
  CUDACHECK(c, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, c->dev));
  CUDACHECK(c, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, interpreterKernel(9, 0, 0), (int)c->prm.threads, 0));
  c->maxCoResident = nsm * nb;
  return mscclSuccess;
}

void freeProgram(mscclProgram* p) {
  if (!p) return;
  DeviceGuard g(p->comm->dev);
  cudaFree(p->dTBs);
  cudaFree(p->dInstr);
  cudaFree(p->dDeps);
  cudaFree(p->dSem);
  cudaFree(p->dScratch);
  delete p;
}

// Debug: per-CTA phase timers of MSCCL_TRACE builds (host-mapped; enabled by env MSCCL_TRACE)
uint64_t* gTraceHost = nullptr;
uint64_t* gTraceDev = nullptr;
uint64_t* traceBuffer() {
  static bool init = false;
  if (!init) {
    init = true;
    const char* v = getenv("MSCCL_TRACE");
    if (v && *v == '1' && cudaHostAlloc(&gTraceHost, 4096 * 32 * sizeof(uint64_t), cudaHostAllocMapped) == cudaSuccess) {
      memset(gTraceHost, 0, 4096 * 32 * sizeof(uint64_t));
      cudaHostGetDevicePointer((void**)&gTraceDev, gTraceHost, 0);
    }
  }
  return gTraceDev;
}

// co-resident CTAs per device for (kernel, threads, dynamic smem); sets the smem attribute
mscclResult_t coResident(mscclComm* c, const void* fn, int threads, int smem, int& out) {
  static std::mutex mu;
  static std::map<std::tuple<const void*, int, int, int>, int> cache;
  std::lock_guard<std::mutex> g(mu);
  auto key = std::make_tuple(fn, threads, smem, c->dev);
  auto it = cache.find(key);
  if (it != cache.end()) {
    out = it->second;
    return mscclSuccess;
  }
  DeviceGuard dg(c->dev);
  if (smem > 48 * 1024) CUDACHECK(c, cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  int nsm = 0, nb = 0;
  CUDACHECK(c, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, c->dev));
  CUDACHECK(c, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, threads, smem));
  out = nsm * nb;
  cache[key] = out;
  return mscclSuccess;
}

// ------------------------------------------------------------------ groups and launches
struct Call {
  mscclComm* comm;
  mscclProgram* prog;
  char* buf[3];
  int dtype, op;
  int64_t n;
  cudaStream_t stream;
};

thread_local int tGroupDepth = 0;
thread_local std::vector<Call> tPending;

struct Geometry {
  int64_t n, E, T;
  int I, cb;
};

// noFifo: every message of the launch is a direct placement (R15), so no FIFO slot bounds
// the tile: T = E (one message per chunk; results do not depend on T, reading R3).
mscclResult_t geometry(mscclComm* c, const mscclProgram* p, int dtype, int64_t n, Geometry& g, bool noFifo = false) {
  const int w = elemBytes(dtype);
  const int V = 16 / w;
  const int R = p->algo.ngpus;
  g.n = n;
  g.cb = p->algo.gpus[0].iChunks / blocksOf(p->algo.coll, BUF_IN, R);
  int64_t e = (n + g.cb - 1) / g.cb;
  g.E = (e + V - 1) / V * V;
  int64_t t;
  if (p->algo.proto == PROTO_LL128)  // whole 128-byte lines (120 payload bytes) per piece
    t = (c->prm.slotBytes / 128 / p->maxCnt) * 120 / w / V * V;
  else
    t = (p->algo.proto == PROTO_LL ? c->prm.slotBytes / 2 : c->prm.slotBytes) / ((int64_t)p->maxCnt * w) / V * V;
  if (t < V) return setErr(c, mscclInvalidUsage, "FIFO slot too small for the program's largest count");
  if (noFifo) t = g.E;
  g.T = std::min<int64_t>(t, g.E);
  g.I = (int)((g.E + g.T - 1) / g.T);
  return mscclSuccess;
}

mscclResult_t ensureScratch(mscclComm* c, mscclProgram* p, size_t bytes) {
  if (bytes <= p->scratchBytes) return mscclSuccess;
  DeviceGuard dg(c->dev);
  CUDACHECK(c, cudaDeviceSynchronize());  // growing scratch: the old one may be in use
  cudaFree(p->dScratch);
  p->dScratch = nullptr;
  p->scratchBytes = 0;
  size_t sz = (bytes + 4095) / 4096 * 4096;
  CUDACHECK(c, cudaMalloc(&p->dScratch, sz));
  p->scratchBytes = sz;
  return mscclSuccess;
}

mscclResult_t launchCalls(std::vector<Call>& calls) {
  // one cooperative launch per device, covering every rank of the group on that device
  std::map<int, std::vector<Call*>> byDev;
  for (auto& cl : calls) byDev[cl.comm->dev].push_back(&cl);
  for (auto& kv : byDev) {
    auto& v = kv.second;
    std::sort(v.begin(), v.end(), [](Call* a, Call* b) { return a->comm->rank < b->comm->rank; });
    mscclComm* c0 = v[0]->comm;
    if ((int)v.size() > MSCCL_MAX_LOCAL) return setErr(c0, mscclInvalidUsage, "too many ranks on one device");
    if (c0->clique) {
      int onDev = 0;
      for (auto* cm : c0->clique->comms)
        if (cm->dev == c0->dev) onDev++;
      if (onDev != (int)v.size())
        return setErr(c0, mscclInvalidUsage,
                      "ranks sharing a GPU must all be called inside one mscclGroupStart/End");
    }
    for (auto* cl : v) {
      if (cl->stream != v[0]->stream) return setErr(cl->comm, mscclInvalidUsage, "ranks on one GPU must use one stream in a group");
      if (cl->prog->index != v[0]->prog->index || cl->dtype != v[0]->dtype || cl->op != v[0]->op || cl->n != v[0]->n)
        return setErr(cl->comm, mscclInvalidUsage, "ranks in a group disagree on program/count/datatype/op");
    }
    mscclProgram* p0 = v[0]->prog;
    // direct placement needs every rank's buffers in this launch (rank r at slot r) and the
    // Simple protocol; one launch covering all ranks also orders it against earlier launches
    const bool useTma = p0->algo.proto == PROTO_SIMPLE && c0->prm.tma && tmaSmemBytes() > 0;
    const bool direct = p0->algo.proto == PROTO_SIMPLE && c0->prm.direct && (int)v.size() == p0->algo.ngpus && !useTma;
    bool noFifo = direct && c0->prm.directTile;
    for (auto* cl : v) noFifo = noFifo && cl->prog->allDirect;
    Geometry g{};
    mscclResult_t r = geometry(c0, p0, v[0]->dtype, v[0]->n, g, noFifo);
    if (r != mscclSuccess) return r;
    KernelArgs ka;
    memset(&ka, 0, sizeof(ka));
    ka.nLocal = (int)v.size();
    ka.I = g.I;
    ka.n = g.n;
    ka.E = g.E;
    ka.T = g.T;
    ka.cb = g.cb;
    ka.slots = (int)c0->prm.slots;
    ka.proto = p0->algo.proto == PROTO_LL ? 1 : (p0->algo.proto == PROTO_LL128 ? 2 : 0);
    ka.slotBytes = c0->prm.slotBytes;
    ka.timeoutNs = (uint64_t)c0->prm.timeoutS * 1000000000ull;
    ka.trace = traceBuffer();
    int cta = 0;
    for (int i = 0; i < (int)v.size(); i++) {
      Call* cl = v[i];
      mscclProgram* p = cl->prog;
      RankArgs& ra = ka.rank[i];
      ra.tbs = p->dTBs;
      ra.instrs = p->dInstr;
      ra.deps = p->dDeps;
      ra.sem = p->dSem;
      ra.gen = p->dSem + p->nTB;
      size_t need = (size_t)p->algo.gpus[cl->comm->rank].sChunks * g.E * elemBytes(cl->dtype);
      r = ensureScratch(cl->comm, p, need);
      if (r != mscclSuccess) return r;
      ra.buf[0] = cl->buf[0];
      ra.buf[1] = cl->buf[1];
      ra.buf[2] = p->dScratch;
      ra.nTB = p->nTB;
      ra.ctaStart = cta;
      ra.abortFlag = (uint32_t*)(cl->comm->region + cl->comm->abortOff());
      ra.hostAbort = cl->comm->hostAbortDev;
      cta += p->nTB;
      if (cl->comm->sysScope) ka.sysScope = 1;
    }
    if (cta == 0) continue;
    // work-balanced placement: thread blocks ordered by the bytes they move (heaviest first,
    // ties by rank then id, so the order is deterministic); block indices are handed to SMs
    // in increasing order, so the heavy blocks land on distinct SMs before any SM gets two
    if (c0->prm.balance && cta <= MSCCL_CTA_MAP && (int)v.size() <= 16) {
      std::vector<std::tuple<int64_t, int, int>> order;
      for (int i = 0; i < (int)v.size(); i++) {
        const mscclProgram* p = v[i]->prog;
        const auto& wk = direct ? p->tbWorkDirect : p->tbWork;
        for (int t = 0; t < p->nTB; t++) order.emplace_back(-wk[t], i, t);
      }
      std::stable_sort(order.begin(), order.end());
      for (size_t k = 0; k < order.size(); k++)
        ka.ctaMap[k] = (uint16_t)((std::get<1>(order[k]) << 12) | std::get<2>(order[k]));
      ka.ctaMapN = (int32_t)order.size();
    }
    const void* fn = p0->hasReduce ? interpreterKernel(v[0]->dtype, v[0]->op, ka.proto)
                                   : copyKernel(elemBytes(v[0]->dtype), ka.proto);
    ka.useTma = useTma ? 1 : 0;
    ka.direct = direct ? 1 : 0;
    ka.warpFlags = (ka.proto == 0 && c0->prm.warp && !ka.useTma) ? 1 : 0;
    ka.prefetch = (ka.proto == 0 && c0->prm.prefetch) ? 1 : 0;
    ka.directHints = (int32_t)c0->prm.directHints;
    const int smem = ka.useTma ? tmaSmemBytes() : 0;
    int maxCta = 0;
    r = coResident(c0, fn, (int)c0->prm.threads, smem, maxCta);
    if (r != mscclSuccess) return r;
    if (cta > maxCta) {
      std::ostringstream o;
      o << "program needs " << cta << " co-resident CTAs on device " << c0->dev << " but at most " << maxCta
        << " fit (use fewer instances/channels, or MSCCL_TMA=0 / fewer MSCCL_THREADS for more CTAs per SM)";
      return setErr(c0, mscclInvalidUsage, o.str());
    }
    DeviceGuard dg(c0->dev);
    void* args[] = {&ka};
    if (debugOn())
      fprintf(stderr, "[msccl] launch dev %d ranks %d program %s ctas %d threads %d n %lld E %lld T %lld I %d\n",
              c0->dev, ka.nLocal, p0->algo.name.c_str(), cta, (int)c0->prm.threads, (long long)g.n,
              (long long)g.E, (long long)g.T, g.I);
    CUDACHECK(c0, cudaLaunchCooperativeKernel(fn, dim3(cta), dim3((unsigned)c0->prm.threads), args, (size_t)smem,
                                              v[0]->stream));
    gLaunches++;
  }
  return mscclSuccess;
}

mscclResult_t enqueue(Call cl) {
  if (tGroupDepth > 0) {
    tPending.push_back(cl);
    return mscclSuccess;
  }
  std::vector<Call> one{cl};
  return launchCalls(one);
}

mscclProgram* selectProgram(mscclComm* c, int coll, size_t bytes) {
  for (auto* p : c->programs) {
    if (p->algo.coll != coll) continue;
    if (bytes < p->minBytes) continue;
    if (p->maxBytes != 0 && bytes >= p->maxBytes) continue;
    return p;
  }
  return nullptr;
}

bool overlaps(const char* a, size_t na, const char* b, size_t nb) { return a < b + nb && b < a + na; }

mscclResult_t runColl(mscclProgram* p, int coll, const void* sendbuff, void* recvbuff, size_t count, int dtype, int op,
                      mscclComm* c, cudaStream_t stream) {
  if (!c) return setErr(nullptr, mscclInvalidArgument, "null communicator");
  if (dtype < 0 || dtype >= mscclNumTypes) return setErr(c, mscclInvalidArgument, "invalid datatype");
  if (op < 0 || op >= mscclNumOps) return setErr(c, mscclInvalidArgument, "invalid reduction op (avg is not supported)");
  if (!c->connected) return setErr(c, mscclInvalidUsage, "communicator not connected (call mscclCommConnect)");
  if (*c->hostAbort) return setErr(c, mscclRemoteError, "communicator aborted by the device watchdog");
  if (count == 0) return mscclSuccess;
  if (!sendbuff || !recvbuff) return setErr(c, mscclInvalidArgument, "null buffer");
  const int w = elemBytes(dtype);
  const int R = c->nranks;
  if (!p) {
    p = selectProgram(c, coll, count * (size_t)w);
    if (!p) {
      std::ostringstream o;
      o << "no loaded program for this collective with " << R << " ranks and " << count * (size_t)w << " bytes";
      return setErr(c, mscclNoMatchingProgram, o.str());
    }
  } else {
    coll = p->algo.coll;
  }
  size_t inElems = count * blocksOf(coll, BUF_IN, R), outElems = count * blocksOf(coll, BUF_OUT, R);
  const char* sb = (const char*)sendbuff;
  char* rb = (char*)recvbuff;
  bool inplace = false;
  if (coll == COLL_ALLREDUCE || coll == COLL_CUSTOM) inplace = sb == rb;
  else if (coll == COLL_ALLGATHER) inplace = sb == rb + (size_t)c->rank * count * w;
  else if (coll == COLL_REDUCESCATTER) inplace = rb == sb + (size_t)c->rank * count * w;
  else if (coll == COLL_ALLTOALL) inplace = false;
  if (!inplace && overlaps(sb, inElems * w, rb, outElems * w))
    return setErr(c, mscclInvalidUsage, "send and receive buffers overlap (and the call is not in NCCL in-place form)");
  Call cl;
  cl.comm = c;
  cl.prog = p;
  cl.dtype = dtype;
  cl.op = op;
  cl.n = (int64_t)count;
  cl.stream = stream;
  if (p->algo.inplace) {
    if (!inplace) {  // reading R8: an in-place program called out of place gets a pre-copy
      DeviceGuard dg(c->dev);
      CUDACHECK(c, cudaMemcpyAsync(rb, sb, inElems * w, cudaMemcpyDeviceToDevice, stream));
    }
    cl.buf[0] = rb;
    cl.buf[1] = rb;
  } else {
    if (inplace && !p->algo.aliassafe)
      return setErr(c, mscclInvalidUsage, "in-place call on an out-of-place program that is not marked aliassafe");
    cl.buf[0] = (char*)sb;
    cl.buf[1] = rb;
  }
  cl.buf[2] = nullptr;
  return enqueue(cl);
}

}  // namespace

// ================================================================== C ABI
extern "C" {

const char* mscclGetErrorString(mscclResult_t r) {
  switch (r) {
    case mscclSuccess: return "no error";
    case mscclUnhandledCudaError: return "unhandled cuda error";
    case mscclSystemError: return "unhandled system error";
    case mscclInternalError: return "internal error";
    case mscclInvalidArgument: return "invalid argument";
    case mscclInvalidUsage: return "invalid usage";
    case mscclRemoteError: return "remote process exited or there was a network error (watchdog)";
    case mscclInProgress: return "operation in progress";
    case mscclInvalidProgram: return "invalid MSCCL-IR program";
    case mscclNoMatchingProgram: return "no loaded program matches the call";
  }
  return "unknown result code";
}

const char* mscclGetLastError(mscclComm_t comm) {
  static thread_local std::string copy;
  std::lock_guard<std::mutex> g(gMu);
  copy = comm ? comm->lastError : gLastError;
  return copy.c_str();
}

mscclResult_t mscclSetParam(const char* key, int64_t value) {
  if (!key) return mscclInvalidArgument;
  currentParams();
  std::lock_guard<std::mutex> g(gMu);
  int64_t* r = paramRef(gParams, key);
  if (!r) return mscclInvalidArgument;
  *r = value;
  return mscclSuccess;
}

mscclResult_t mscclGetParam(const char* key, int64_t* value) {
  if (!key || !value) return mscclInvalidArgument;
  Params p = currentParams();
  int64_t* r = paramRef(p, key);
  if (!r) return mscclInvalidArgument;
  *value = *r;
  return mscclSuccess;
}

uint64_t mscclLaunchCount(void) { return gLaunches.load(); }

// not part of msccl.h: debug access to the MSCCL_TRACE phase timers (4096 CTAs x 8)
uint64_t* msccl_debug_trace(void) { return gTraceHost; }

mscclResult_t mscclCommInitAll(mscclComm_t* comms, int ndev, const int* devlist) {
  if (!comms || ndev < 1) return setErr(nullptr, mscclInvalidArgument, "bad arguments to mscclCommInitAll");
  auto clique = std::make_shared<Clique>();
  for (int i = 0; i < ndev; i++) {
    mscclComm* c = new mscclComm();
    c->nranks = ndev;
    c->rank = i;
    c->dev = devlist ? devlist[i] : i;
    c->clique = clique;
    mscclResult_t r = allocRegion(c);
    if (r != mscclSuccess) {
      for (auto* x : clique->comms) mscclCommDestroy(x);
      delete c;
      return r;
    }
    clique->comms.push_back(c);
  }
  for (auto* c : clique->comms) {
    for (auto* p : clique->comms) {
      c->peerBase[p->rank] = p->region;
      if (p->dev != c->dev) {
        c->sysScope = true;
        int can = 0;
        cudaDeviceCanAccessPeer(&can, c->dev, p->dev);
        if (!can) return setErr(c, mscclSystemError, "no peer access between devices");
        DeviceGuard g(c->dev);
        cudaError_t e = cudaDeviceEnablePeerAccess(p->dev, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
          return setErr(c, mscclUnhandledCudaError, std::string("cudaDeviceEnablePeerAccess: ") + cudaGetErrorString(e));
        cudaGetLastError();
      }
    }
    c->connected = true;
  }
  for (int i = 0; i < ndev; i++) comms[i] = clique->comms[i];
  return mscclSuccess;
}

mscclResult_t mscclCommInitRank(mscclComm_t* comm, int nranks, int rank, int cudaDev) {
  if (!comm || nranks < 1 || rank < 0 || rank >= nranks) return setErr(nullptr, mscclInvalidArgument, "bad arguments to mscclCommInitRank");
  mscclComm* c = new mscclComm();
  c->nranks = nranks;
  c->rank = rank;
  c->dev = cudaDev;
  mscclResult_t r = allocRegion(c);
  if (r != mscclSuccess) {
    delete c;
    return r;
  }
  if (nranks == 1) c->connected = true;
  *comm = c;
  return mscclSuccess;
}

mscclResult_t mscclCommExportHandle(mscclComm_t c, void* handle, size_t* bytes) {
  if (!c || !handle) return setErr(c, mscclInvalidArgument, "null argument");
  memset(handle, 0, MSCCL_HANDLE_BYTES);
  DeviceGuard g(c->dev);
  cudaIpcMemHandle_t h;
  CUDACHECK(c, cudaIpcGetMemHandle(&h, c->region));
  static_assert(sizeof(h) + 32 <= MSCCL_HANDLE_BYTES, "handle size");
  memcpy(handle, &h, sizeof(h));
  // parameters that both ends of a connection must agree on (region layout, warp partition)
  int64_t meta[4] = {(int64_t)c->regionBytes, (int64_t)c->dev, c->prm.threads, c->prm.warp};
  memcpy((char*)handle + sizeof(h), meta, sizeof(meta));
  if (bytes) *bytes = MSCCL_HANDLE_BYTES;
  return mscclSuccess;
}

mscclResult_t mscclCommConnect(mscclComm_t c, const void* allHandles) {
  if (!c || !allHandles) return setErr(c, mscclInvalidArgument, "null argument");
  if (c->connected) return mscclSuccess;
  DeviceGuard g(c->dev);
  for (int p = 0; p < c->nranks; p++) {
    if (p == c->rank) continue;
    const char* h = (const char*)allHandles + (size_t)p * MSCCL_HANDLE_BYTES;
    cudaIpcMemHandle_t ih;
    memcpy(&ih, h, sizeof(ih));
    int64_t meta[4];
    memcpy(meta, h + sizeof(ih), sizeof(meta));
    if ((size_t)meta[0] != c->regionBytes) return setErr(c, mscclInvalidUsage, "peer region size differs (ranks use different MSCCL_* parameters)");
    if (meta[2] != c->prm.threads || meta[3] != c->prm.warp)
      return setErr(c, mscclInvalidUsage, "peer uses different MSCCL_THREADS / MSCCL_WARP_FLAGS (the warp partition must match)");
    void* ptr = nullptr;
    CUDACHECK(c, cudaIpcOpenMemHandle(&ptr, ih, cudaIpcMemLazyEnablePeerAccess));
    c->peerBase[p] = (char*)ptr;
    c->peerIpc[p] = true;
    c->sysScope = true;
  }
  c->connected = true;
  return mscclSuccess;
}

mscclResult_t mscclCommDestroy(mscclComm_t c) {
  if (!c) return mscclSuccess;
  {
    DeviceGuard g(c->dev);
    cudaDeviceSynchronize();
    for (auto* p : c->programs) freeProgram(p);
    c->programs.clear();
    for (int p = 0; p < c->nranks; p++)
      if (c->peerIpc[p]) cudaIpcCloseMemHandle(c->peerBase[p]);
    cudaFree(c->region);
    cudaFreeHost(c->hostAbort);
  }
  if (c->clique) {
    auto& v = c->clique->comms;
    v.erase(std::remove(v.begin(), v.end(), c), v.end());
  }
  delete c;
  return mscclSuccess;
}

mscclResult_t mscclCommCount(const mscclComm_t c, int* count) {
  if (!c || !count) return mscclInvalidArgument;
  *count = c->nranks;
  return mscclSuccess;
}
mscclResult_t mscclCommUserRank(const mscclComm_t c, int* rank) {
  if (!c || !rank) return mscclInvalidArgument;
  *rank = c->rank;
  return mscclSuccess;
}
mscclResult_t mscclCommCuDevice(const mscclComm_t c, int* device) {
  if (!c || !device) return mscclInvalidArgument;
  *device = c->dev;
  return mscclSuccess;
}

mscclResult_t mscclCommGetAsyncError(mscclComm_t c, mscclResult_t* err) {
  if (!c || !err) return mscclInvalidArgument;
  *err = (*(volatile uint32_t*)c->hostAbort) ? mscclRemoteError : mscclSuccess;
  return mscclSuccess;
}

mscclResult_t mscclValidateProgram(const char* ir, size_t irBytes, int nranks, int slots, int maxTbs, char* err,
                                   size_t errBytes) {
  if (err && errBytes) err[0] = 0;
  if (!ir) return mscclInvalidArgument;
  try {
    Algo a = parseIR(ir, irBytes);
    Params prm = currentParams();
    validateIR(a, nranks, slots > 0 ? slots : (int)prm.slots, maxTbs > 0 ? maxTbs : 148, (int)prm.maxChannels);
  } catch (const IRError& e) {
    if (err && errBytes) {
      strncpy(err, e.what(), errBytes - 1);
      err[errBytes - 1] = 0;
    }
    setErr(nullptr, mscclInvalidProgram, e.what());
    return mscclInvalidProgram;
  }
  return mscclSuccess;
}

mscclResult_t mscclLoadProgram(mscclComm_t c, const char* ir, size_t irBytes, size_t minBytes, size_t maxBytes,
                               mscclProgram_t* out) {
  if (!c || !ir || !out) return setErr(c, mscclInvalidArgument, "null argument");
  if (!c->connected) return setErr(c, mscclInvalidUsage, "communicator not connected (call mscclCommConnect first)");
  std::unique_ptr<mscclProgram> p(new mscclProgram());
  p->comm = c;
  try {
    p->algo = parseIR(ir, irBytes);
    validateIR(p->algo, c->nranks, (int)c->prm.slots, std::min(c->maxCoResident, 1 << 15), (int)c->prm.maxChannels);
  } catch (const IRError& e) {
    return setErr(c, mscclInvalidProgram, e.what());
  }
  p->minBytes = minBytes;
  p->maxBytes = maxBytes;
  p->maxCnt = p->algo.maxCnt();
  p->hasReduce = p->algo.hasReduce();
  const GpuProgram& g = p->algo.gpus[c->rank];
  p->nTB = (int)g.tbs.size();
  const DirectInfo dinfo = directPlacement(p->algo, c->rank);
  std::vector<DevTB> tbs(p->nTB);
  p->tbWork.assign(p->nTB, 0);
  p->tbWorkDirect.assign(p->nTB, 0);
  std::vector<DevInstr> ins;
  std::vector<uint64_t> deps;
  for (int t = 0; t < p->nTB; t++) {
    const ThreadBlock& tb = g.tbs[t];
    DevTB& d = tbs[t];
    memset(&d, 0, sizeof(d));
    d.nSteps = (int)tb.steps.size();
    d.instrStart = (uint32_t)ins.size();
    d.tbId = tb.id;
    d.sendPeer = tb.send;
    if (tb.send >= 0) {
      d.sendFifo = c->peerBase[tb.send] + c->fifoOff(c->rank, tb.chan);
      d.sendHead = (uint64_t*)(c->peerBase[tb.send] + c->flagOff(0, c->rank, tb.chan));
      d.sendAck = (uint64_t*)(c->region + c->flagOff(1, tb.send, tb.chan));
      d.sendCnt = (uint64_t*)(c->region + c->flagOff(2, tb.send, tb.chan));
    }
    if (tb.recv >= 0) {
      d.recvFifo = c->region + c->fifoOff(tb.recv, tb.chan);
      d.recvHead = (uint64_t*)(c->region + c->flagOff(0, tb.recv, tb.chan));
      d.recvAck = (uint64_t*)(c->peerBase[tb.recv] + c->flagOff(1, c->rank, tb.chan));
      d.recvCnt = (uint64_t*)(c->region + c->flagOff(3, tb.recv, tb.chan));
    }
    for (size_t si = 0; si < tb.steps.size(); si++) {
      const Instr& in = tb.steps[si];
      DevInstr di;
      memset(&di, 0, sizeof(di));
      di.op = (uint8_t)in.op;
      di.srcBuf = (uint8_t)(in.srcBuf == BUF_NONE ? 0 : in.srcBuf);
      di.dstBuf = (uint8_t)(in.dstBuf == BUF_NONE ? 0 : in.dstBuf);
      if (in.deps.size() > 255) return setErr(c, mscclInvalidProgram, "V8: more than 255 dependencies on one step");
      di.nDeps = (uint8_t)in.deps.size();
      di.cnt = (uint16_t)in.cnt;
      di.hasDep = in.hasDep ? 1 : 0;
      di.srcOff = (uint32_t)std::max(in.srcOff, 0);
      di.dstOff = (uint32_t)std::max(in.dstOff, 0);
      di.depStart = (uint32_t)deps.size();
      // dependency word: the waiter computes the semaphore target without reading the
      // other thread block's descriptor (one memory round trip instead of two)
      for (auto& dp : in.deps)
        deps.push_back(((uint64_t)dp.first << 48) | ((uint64_t)dp.second << 32) |
                       (uint64_t)(uint32_t)g.tbs[dp.first].steps.size());
      if (dinfo.recvDirect[t][si]) di.flags |= DI_RECV_DIRECT;
      {  // operand touches of this instruction (mscclProgramTouches costs)
        static const int cost[OP_COUNT] = {0, 2, 2, 2, 3, 3, 3, 4, 3};
        int cd = cost[in.op];
        if (dinfo.recvDirect[t][si]) cd = in.op == OP_RCS ? 2 : 0;
        p->tbWork[t] += (int64_t)cost[in.op] * in.cnt;
        p->tbWorkDirect[t] += (int64_t)cd * in.cnt;
      }
      const bool sends = in.op == OP_SEND || in.op == OP_RRS || in.op == OP_RRCS || in.op == OP_RCS;
      if (sends && !dinfo.sendDirect[t][si]) p->allDirect = false;
      if (dinfo.sendDirect[t][si]) {
        di.flags |= DI_SEND_DIRECT;
        di.rdstBuf = (uint8_t)dinfo.rdstBuf[t][si];
        di.rdstOff = (uint32_t)dinfo.rdstOff[t][si];
        if (dinfo.rterminal[t][si]) di.flags |= DI_SEND_TERMINAL;
      }
      ins.push_back(di);
    }
    // reading R16: mark runs [cpy ->D] re ->D re ->D ... (same D and cnt, no hasDep before the
    // last member, sources distinct from D) as one fused chain for the interpreter
    size_t base = d.instrStart;
    for (size_t s0 = 0; s0 < tb.steps.size();) {
      const Instr& h = tb.steps[s0];
      size_t e = s0;
      if (h.op == OP_COPY || h.op == OP_REDUCE) {
        auto sameDst = [&](const Instr& x) {
          return x.op == OP_REDUCE && x.dstBuf == h.dstBuf && x.dstOff == h.dstOff && x.cnt == h.cnt &&
                 !(x.srcBuf == h.dstBuf && x.srcOff < h.dstOff + h.cnt && h.dstOff < x.srcOff + x.cnt);
        };
        bool headOk = !(h.srcBuf == h.dstBuf && h.srcOff < h.dstOff + h.cnt && h.dstOff < h.srcOff + h.cnt);
        if (headOk && !h.hasDep) {
          e = s0 + 1;
          while (e < tb.steps.size() && e - s0 < 16 && sameDst(tb.steps[e])) {
            if (tb.steps[e].hasDep) {
              e++;
              break;
            }
            e++;
          }
        }
      }
      size_t len = e > s0 ? e - s0 : 1;
      if (len >= 2) {
        ins[base + s0].flags |= DI_CHAIN_HEAD;
        ins[base + s0].chainLen = (uint16_t)len;
      }
      s0 += len;
    }
  }
  p->nInstr = (int)ins.size();
  DeviceGuard dg(c->dev);
  if (p->nTB) {
    CUDACHECK(c, cudaMalloc(&p->dTBs, tbs.size() * sizeof(DevTB)));
    CUDACHECK(c, cudaMemcpy(p->dTBs, tbs.data(), tbs.size() * sizeof(DevTB), cudaMemcpyHostToDevice));
    CUDACHECK(c, cudaMalloc(&p->dSem, 2 * p->nTB * sizeof(uint64_t)));
    CUDACHECK(c, cudaMemset(p->dSem, 0, 2 * p->nTB * sizeof(uint64_t)));
  }
  if (!ins.empty()) {
    CUDACHECK(c, cudaMalloc(&p->dInstr, ins.size() * sizeof(DevInstr)));
    CUDACHECK(c, cudaMemcpy(p->dInstr, ins.data(), ins.size() * sizeof(DevInstr), cudaMemcpyHostToDevice));
  }
  if (!deps.empty()) {
    CUDACHECK(c, cudaMalloc(&p->dDeps, deps.size() * sizeof(uint64_t)));
    CUDACHECK(c, cudaMemcpy(p->dDeps, deps.data(), deps.size() * sizeof(uint64_t), cudaMemcpyHostToDevice));
  }
  p->index = (int)c->programs.size();
  c->programs.push_back(p.get());
  *out = p.release();
  return mscclSuccess;
}

mscclResult_t mscclUnloadProgram(mscclComm_t c, mscclProgram_t p) {
  if (!c || !p) return mscclInvalidArgument;
  auto it = std::find(c->programs.begin(), c->programs.end(), p);
  if (it == c->programs.end()) return setErr(c, mscclInvalidArgument, "program not loaded on this communicator");
  c->programs.erase(it);
  {
    DeviceGuard g(c->dev);
    cudaDeviceSynchronize();
  }
  freeProgram(p);
  return mscclSuccess;
}

mscclResult_t mscclProgramInfo(mscclProgram_t p, int* nTB, int* nInstr, int* inplace) {
  if (!p) return mscclInvalidArgument;
  if (nTB) *nTB = p->nTB;
  if (nInstr) *nInstr = p->nInstr;
  if (inplace) *inplace = p->algo.inplace ? 1 : 0;
  return mscclSuccess;
}

mscclResult_t mscclProgramTouches(mscclProgram_t p, int direct, int64_t* touches) {
  if (!p || !touches) return mscclInvalidArgument;
  static const int cost[OP_COUNT] = {0, 2, 2, 2, 3, 3, 3, 4, 3};
  const DirectInfo di = directPlacement(p->algo, p->comm->rank);
  int64_t n = 0;
  const GpuProgram& g = p->algo.gpus[p->comm->rank];
  for (size_t t = 0; t < g.tbs.size(); t++)
    for (size_t s = 0; s < g.tbs[t].steps.size(); s++) {
      const Instr& in = g.tbs[t].steps[s];
      int c = cost[in.op];
      if (direct && di.recvDirect[t][s]) c = in.op == OP_RCS ? 2 : 0;
      n += (int64_t)c * in.cnt;
    }
  *touches = n;
  return mscclSuccess;
}

mscclResult_t mscclAllReduce(const void* s, void* r, size_t count, mscclDataType_t dt, mscclRedOp_t op, mscclComm_t c,
                             mscclStream_t st) {
  return runColl(nullptr, COLL_ALLREDUCE, s, r, count, dt, op, c, (cudaStream_t)st);
}
mscclResult_t mscclAllGather(const void* s, void* r, size_t count, mscclDataType_t dt, mscclComm_t c, mscclStream_t st) {
  return runColl(nullptr, COLL_ALLGATHER, s, r, count, dt, mscclSum, c, (cudaStream_t)st);
}
mscclResult_t mscclReduceScatter(const void* s, void* r, size_t count, mscclDataType_t dt, mscclRedOp_t op,
                                 mscclComm_t c, mscclStream_t st) {
  return runColl(nullptr, COLL_REDUCESCATTER, s, r, count, dt, op, c, (cudaStream_t)st);
}
mscclResult_t mscclAllToAll(const void* s, void* r, size_t count, mscclDataType_t dt, mscclComm_t c, mscclStream_t st) {
  return runColl(nullptr, COLL_ALLTOALL, s, r, count, dt, mscclSum, c, (cudaStream_t)st);
}
mscclResult_t mscclRunProgram(mscclProgram_t p, const void* s, void* r, size_t count, mscclDataType_t dt,
                              mscclRedOp_t op, mscclComm_t c, mscclStream_t st) {
  if (!p) return setErr(c, mscclInvalidArgument, "null program");
  if (p->comm != c) return setErr(c, mscclInvalidArgument, "program was loaded on another communicator");
  return runColl(p, p->algo.coll, s, r, count, dt, op, c, (cudaStream_t)st);
}

mscclResult_t mscclGroupStart(void) {
  tGroupDepth++;
  return mscclSuccess;
}

mscclResult_t mscclGroupEnd(void) {
  if (tGroupDepth <= 0) return setErr(nullptr, mscclInvalidUsage, "mscclGroupEnd without mscclGroupStart");
  if (--tGroupDepth > 0) return mscclSuccess;
  std::vector<Call> calls;
  calls.swap(tPending);
  if (calls.empty()) return mscclSuccess;
  return launchCalls(calls);
}

}  // extern "C"
