// Host runtime behind include/msccl.h: communicators, shared regions, program loading,
// program selection by size range (MSCCLang §6), geometry, launch.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <set>
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

// Library defaults = the tuned configuration: 4 x 256 KiB Simple slots, 256
// threads per CTA (2 CTAs per SM), direct placement on. LL / LL128 have their own FIFO slots.
struct Params {
  int64_t slots = 4, slotBytes = 262144, llSlotBytes = 65536, ll128SlotBytes = 262144, maxChannels = 32,
          threads = 256, timeoutS = 60, direct = 1, directTile = 1, directHints = 25, regMax = 64,
          crossLaunch = 0;
};

std::mutex gMu;
Params gParams;
bool gEnvRead = false;
std::string gLastError;
std::atomic<uint64_t> gLaunches{0};

int64_t* paramRef(Params& p, const std::string& k) {
  if (k == "MSCCL_SLOTS") return &p.slots;
  if (k == "MSCCL_SLOT_BYTES") return &p.slotBytes;
  if (k == "MSCCL_LL_SLOT_BYTES") return &p.llSlotBytes;
  if (k == "MSCCL_LL128_SLOT_BYTES") return &p.ll128SlotBytes;
  if (k == "MSCCL_MAX_REGISTRATIONS") return &p.regMax;
  if (k == "MSCCL_MAX_CHANNELS") return &p.maxChannels;
  if (k == "MSCCL_THREADS") return &p.threads;
  if (k == "MSCCL_TIMEOUT_S") return &p.timeoutS;
  if (k == "MSCCL_DIRECT") return &p.direct;
  if (k == "MSCCL_DIRECT_TILE") return &p.directTile;
  if (k == "MSCCL_DIRECT_HINTS") return &p.directHints;
  if (k == "MSCCL_CROSS_LAUNCH") return &p.crossLaunch;
  return nullptr;
}

Params currentParams() {
  std::lock_guard<std::mutex> g(gMu);
  if (!gEnvRead) {
    gEnvRead = true;
    for (const char* k : {"MSCCL_SLOTS", "MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES",
                          "MSCCL_MAX_CHANNELS", "MSCCL_THREADS", "MSCCL_TIMEOUT_S", "MSCCL_DIRECT",
                          "MSCCL_DIRECT_TILE", "MSCCL_DIRECT_HINTS", "MSCCL_MAX_REGISTRATIONS", "MSCCL_CROSS_LAUNCH"}) {
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

// A registered user buffer (reading R15b): peers of a CUDA-IPC communicator can place messages
// straight into it. Registration index = position in the comm's table (same on every rank when
// every rank registers in the same order, but each rank publishes its own index anyway).
struct mscclReg {
  mscclComm* comm = nullptr;
  int idx = -1;
  char* base = nullptr;      // registered range [base, base + size) in this process
  size_t size = 0;
  bool connected = false;    // mscclRegConnect done: every peer's matching buffer is mapped
  char* allocBase = nullptr;  // the device allocation holding the range (what CUDA IPC exports)
  std::vector<char*> peerMapped;  // IPC mappings this rank uses for peers' buffer `idx` (allocation bases)
  std::vector<std::pair<int, std::string>> peerKeys;  // their ipcCache entries
};

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
  uint64_t launchesDirect1 = 0, launchesDirect2 = 0;  // launches this rank took part in, by direct mode
  uint64_t depthChecks = 0;            // V9 re-runs at a launch's real pipeline depth (R24)
  uint32_t loadCounter = 0;            // programs loaded so far (multimem group-barrier epochs)
  // NVLS buffers (mscclNvlsAlloc): this rank's unicast range and the multicast address of it
  struct Nvls {
    char* uc;
    char* mc;
    size_t size;
    unsigned long long phys;     // CUmemGenericAllocationHandle of this rank's memory
    unsigned long long mcHandle; // the multicast object (shared by the clique)
    bool owner;                  // this rank maps / releases the multicast VA
  };
  std::vector<Nvls> nvls;
  char** dPeerRegion = nullptr;        // device [nranks]: every rank's region in this address space
  std::vector<mscclReg*> regs;         // by index (nullptr = free)
  char** dRegMap = nullptr;            // device [nranks][regMax]: peers' registered buffers, mapped here
  std::vector<char*> hRegMap;
  // opened peer allocations (CUDA IPC handles can be opened once per process): refcounted
  std::map<std::pair<int, std::string>, std::pair<char*, int>> ipcCache;

  // region layout: one receiver-side FIFO per protocol (Simple, LL, LL128), each
  // [src rank][channel][slot] x that protocol's slot bytes, then the flag lines
  int64_t protoSlotBytes(int proto) const {
    return proto == PROTO_LL ? prm.llSlotBytes : proto == PROTO_LL128 ? prm.ll128SlotBytes : prm.slotBytes;
  }
  size_t fifoBase(int proto) const {
    size_t off = 0;
    for (int p = 0; p < proto; p++) off += (size_t)nranks * prm.maxChannels * prm.slots * protoSlotBytes(p);
    return off;
  }
  size_t fifoOff(int proto, int src, int ch) const {
    return fifoBase(proto) + ((size_t)src * prm.maxChannels + ch) * prm.slots * protoSlotBytes(proto);
  }
  // kind: 0 head, 1 ack, 2 sendCnt, 3 recvCnt, 4 ready (line of the SENDER's region, written by
  // the receiver); one 128-byte line each
  size_t flagOff(int kind, int peer, int ch) const {
    return flagsOff + (((size_t)kind * nranks + peer) * prm.maxChannels + ch) * MSCCL_FLAG_STRIDE * sizeof(uint64_t);
  }
  size_t abortOff() const { return flagOff(5, 0, 0); }
  size_t statsOff() const { return abortOff() + 128; }
  // multimem group-barrier lines (reading R23): [start|done][thread block][source rank]
  size_t mmLineOff() const { return statsOff() + 128; }
  size_t mmBytes() const { return (size_t)2 * MSCCL_MM_MAX_TB * nranks * 128; }
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
  std::vector<char*> retiredScratch;  // outgrown scratch buffers: a captured graph may still use them
  char* dRec = nullptr;    // latency kernels: per-block records (DevTB + instructions), see RankArgs
  int64_t recStride = 0;
  int maxCnt = 1;
  bool hasReduce = false;
  bool allDirect = true;  // every message of this rank's program is a direct placement (R15)
  std::set<int> v9Iters;  // pipeline depths I at which V9 (deadlock freedom) has been verified
  bool hasMultimem = false;
  bool forwards = false;  // some instruction forwards what it received (rcs / rrs / rrcs)
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
  for (int64_t b : {c->prm.slotBytes, c->prm.llSlotBytes, c->prm.ll128SlotBytes})
    if (b < 4096 || b % 256)
      return setErr(c, mscclInvalidArgument, "MSCCL_SLOT_BYTES / MSCCL_LL_SLOT_BYTES / MSCCL_LL128_SLOT_BYTES must be multiples of 256, >= 4096");
  if (c->prm.threads < 64 || c->prm.threads > MSCCL_MAX_THREADS || c->prm.threads % 32) {
    std::ostringstream o;
    o << "MSCCL_THREADS must be a multiple of 32 in 64.." << MSCCL_MAX_THREADS;
    return setErr(c, mscclInvalidArgument, o.str());
  }
  if (c->prm.maxChannels < 1 || c->prm.maxChannels > 1024) return setErr(c, mscclInvalidArgument, "MSCCL_MAX_CHANNELS out of range");
  if (c->prm.regMax < 1 || c->prm.regMax > (1 << 20)) return setErr(c, mscclInvalidArgument, "MSCCL_MAX_REGISTRATIONS out of range");
  DeviceGuard g(c->dev);
  c->fifoBytes = c->fifoBase(3);
  c->flagsOff = c->fifoBytes;
  c->regionBytes = c->mmLineOff() + c->mmBytes();
  CUDACHECK(c, cudaMalloc(&c->region, c->regionBytes));
  CUDACHECK(c, cudaMemset(c->region, 0, c->regionBytes));
  c->hRegMap.assign((size_t)c->nranks * c->prm.regMax, nullptr);
  CUDACHECK(c, cudaMalloc(&c->dRegMap, c->hRegMap.size() * sizeof(char*)));
  CUDACHECK(c, cudaMemset(c->dRegMap, 0, c->hRegMap.size() * sizeof(char*)));
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
  cudaFree(p->dRec);
  for (char* x : p->retiredScratch) cudaFree(x);
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

// the device copy of peerBase (multimem group barriers address every rank's region)
mscclResult_t uploadPeerRegions(mscclComm* c) {
  DeviceGuard g(c->dev);
  if (!c->dPeerRegion) CUDACHECK(c, cudaMalloc(&c->dPeerRegion, c->nranks * sizeof(char*)));
  CUDACHECK(c, cudaMemcpy(c->dPeerRegion, c->peerBase.data(), c->nranks * sizeof(char*), cudaMemcpyHostToDevice));
  return mscclSuccess;
}

// drop a registration: unpublish it and close the peer mappings nobody else uses
void releaseReg(mscclComm* c, mscclReg* r) {
  for (auto& k : r->peerKeys) {
    auto it = c->ipcCache.find(k);
    if (it != c->ipcCache.end() && --it->second.second == 0) {
      cudaIpcCloseMemHandle(it->second.first);
      c->ipcCache.erase(it);
    }
  }
  if (r->idx >= 0 && r->idx < (int)c->regs.size()) {
    c->regs[r->idx] = nullptr;
    for (int p = 0; p < c->nranks; p++) c->hRegMap[(size_t)p * c->prm.regMax + r->idx] = nullptr;
    cudaMemcpy(c->dRegMap, c->hRegMap.data(), c->hRegMap.size() * sizeof(char*), cudaMemcpyHostToDevice);
  }
  delete r;
}

// ------------------------------------------------------------------ groups and launches
struct Call {
  mscclComm* comm;
  mscclProgram* prog;
  char* buf[3];
  int dtype, op;
  int64_t n;
  cudaStream_t stream;
  bool aliased;  // in-place call of an out-of-place (aliassafe) program: no direct placement
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
  const int64_t sb = c->protoSlotBytes(p->algo.proto);
  if (p->algo.proto == PROTO_LL128)  // whole 128-byte lines (120 payload bytes) per piece
    t = (sb / 128 / p->maxCnt) * 120 / w / V * V;
  else
    t = (p->algo.proto == PROTO_LL ? sb / 2 : sb) / ((int64_t)p->maxCnt * w) / V * V;
  if (t < V) return setErr(c, mscclInvalidUsage, "FIFO slot too small for the program's largest count");
  if (noFifo) t = g.E;
  g.T = std::min<int64_t>(t, g.E);
  g.I = (int)((g.E + g.T - 1) / g.T);
  return mscclSuccess;
}

// Scratch (SURVEY §8(b) Ownership): pre-sized at mscclLoadProgram for the program's maxBytes,
// so calls inside that size range never allocate and can be captured in a CUDA graph. A
// program loaded without a maxBytes grows its scratch on the first (uncaptured) call that needs
// more; the outgrown buffer is kept until the program is unloaded, because kernels already
// queued, or graphs captured earlier, still reference it. No host synchronisation either way.
mscclResult_t ensureScratch(mscclComm* c, mscclProgram* p, size_t bytes, cudaStream_t stream) {
  if (bytes <= p->scratchBytes) return mscclSuccess;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  CUDACHECK(c, cudaStreamIsCapturing(stream, &cs));
  if (cs != cudaStreamCaptureStatusNone) {
    std::ostringstream o;
    o << "program '" << p->algo.name << "' needs " << bytes << " bytes of scratch but has " << p->scratchBytes
      << " while the stream is being captured: load it with maxBytes covering this call (scratch is then "
         "pre-sized) or run one uncaptured call of this size first";
    return setErr(c, mscclInvalidUsage, o.str());
  }
  DeviceGuard dg(c->dev);
  size_t sz = (bytes + 4095) / 4096 * 4096;
  char* nb = nullptr;
  CUDACHECK(c, cudaMalloc(&nb, sz));
  if (p->dScratch) p->retiredScratch.push_back(p->dScratch);
  p->dScratch = nb;
  p->scratchBytes = sz;
  return mscclSuccess;
}

// V9 at the launch's real pipeline depth: the loader checked
// 2 iterations; the first call with a deeper pipeline re-runs the abstract machine with I
// iterations and the program remembers the verdict per I.
mscclResult_t checkDepth(mscclComm* c, mscclProgram* p, int I) {
  if (I <= 2 || p->v9Iters.count(I)) return mscclSuccess;
  try {
    deadlockCheckIR(p->algo, (int)c->prm.slots, I);
  } catch (const IRError& e) {
    return setErr(c, mscclInvalidProgram, std::string(e.what()) + " (pipeline depth I=" + std::to_string(I) + ")");
  }
  p->v9Iters.insert(I);
  c->depthChecks++;
  return mscclSuccess;
}

// how a sender reaches [p, p+bytes) of rank c in this call (reading R15b): a raw pointer when
// every rank lives in this process (peer access / virtual ranks), else a registered buffer
uint64_t bufferRef(mscclComm* c, const char* p, size_t bytes) {
  if (!p) return 0;
  if (c->clique) return (uint64_t)(uintptr_t)p;
  for (auto* r : c->regs)
    if (r && r->connected && p >= r->base && p + bytes <= r->base + r->size)
      return MSCCL_REF_REG | ((uint64_t)r->idx << 40) | (uint64_t)(p - r->base);
  return 0;
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
    // one call per communicator per launch: two calls on one comm would share its connection
    // counters, semaphores and FIFOs inside one grid (NCCL aggregates such calls; here it is an error)
    for (size_t i = 1; i < v.size(); i++)
      if (v[i]->comm == v[i - 1]->comm || v[i]->comm->rank == v[i - 1]->comm->rank)
        return setErr(v[i]->comm, mscclInvalidUsage,
                      "two collectives on one communicator (or rank) inside one mscclGroupStart/End");
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
    const int R = p0->algo.ngpus;
    // Direct placement (reading R15) needs the Simple protocol. Mode 1: every rank 0..R-1 of the
    // program is in this launch exactly once (slot r = rank r), so the sender reaches the
    // receiver's buffers through this launch's arguments. Mode 2 (reading R15b): some ranks run
    // in other launches or processes; each connection does a ready handshake per launch.
    bool allHere = (int)v.size() == R;
    for (int i = 0; allHere && i < (int)v.size(); i++) allHere = v[i]->comm->rank == i && v[i]->comm->nranks == R;
    // MSCCL_CROSS_LAUNCH=1 (test mode): run the cross-launch protocol (R15b ready handshakes, R23
    // group barriers, system-scope fences and flags) although every rank is in this one
    // cooperative launch -- the device code of the multi-GPU / multi-process deployment, with
    // all ranks co-resident (so nothing waits on a kernel that might not be running)
    const bool emulateCross = c0->prm.crossLaunch != 0;
    if (emulateCross) allHere = false;
    int direct = 0;
    if (p0->algo.proto == PROTO_SIMPLE && c0->prm.direct) direct = allHere ? 1 : 2;
    bool aliasedAny = false;
    for (auto* cl : v) aliasedAny = aliasedAny || cl->aliased;
    if (direct == 1 && aliasedAny) direct = 0;  // ADVICE: in-place call of an out-of-place program
    // multimem ops (reading R23): buffers of every rank from this launch (mode 1) or through the
    // group barrier's published references (mode 2)
    const int mm = p0->hasMultimem ? (allHere ? 1 : 2) : 0;
    if (mm && v[0]->op == mscclProd && p0->hasReduce)
      return setErr(c0, mscclInvalidArgument, "multimem reductions support sum/max/min (no product, reading R23)");
    // reading R19: one tile per chunk when no message uses a FIFO slot -- unless a rank forwards
    // what it receives (ring AllGather: rcs reads the chunk its predecessor just stored): then
    // the slot-sized tile bounds the data in flight so the forwarded tile is still in L2 when
    // it is read (measured: ring AllGather 337 -> 389 GB/s busBW on 8 virtual ranks)
    bool noFifo = (direct == 1 || direct == 2) && c0->prm.directTile;
    for (auto* cl : v) noFifo = noFifo && cl->prog->allDirect && !cl->prog->forwards;
    // Cross-launch (R15b): whether a message is direct is settled per connection at the ready
    // handshake, so one tile per chunk also needs every destination of this rank reachable by
    // its senders (user buffers inside registrations, or raw pointers in one process; the
    // library's scratch only in one process). Ranks decide from their own buffers; the
    // receiver publishes its tile size on the ready line and a sender whose tile differs (a rank
    // registered differently) raises the watchdog abort instead of storing past a FIFO slot.
    // Across processes this needs every rank to have registered its buffers, so it is opt-in
    // there (MSCCL_DIRECT_TILE=2); in one process every buffer is reachable by construction.
    if (noFifo && direct == 2 && !c0->clique && c0->prm.directTile < 2) noFifo = false;
    if (noFifo && direct == 2) {
      for (auto* cl : v) {
        const int Rr = cl->comm->nranks, w = elemBytes(cl->dtype);
        const size_t inB = (size_t)cl->n * blocksOf(cl->prog->algo.coll, BUF_IN, Rr) * w;
        const size_t outB = (size_t)cl->n * blocksOf(cl->prog->algo.coll, BUF_OUT, Rr) * w;
        const bool sc = cl->prog->algo.gpus[cl->comm->rank].sChunks > 0;
        noFifo = noFifo && !cl->aliased && bufferRef(cl->comm, cl->buf[0], inB) && bufferRef(cl->comm, cl->buf[1], outB) &&
                 (!sc || cl->comm->clique);
      }
    }
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
    ka.slotBytes = c0->protoSlotBytes(p0->algo.proto);
    ka.timeoutNs = c0->prm.timeoutS > 0 ? (uint64_t)c0->prm.timeoutS * 1000000000ull : 0;  // <= 0: no watchdog
    ka.trace = traceBuffer();
    ka.direct = direct;
    ka.tileIsChunk = noFifo ? 1 : 0;
    ka.directHints = (int32_t)c0->prm.directHints;
    ka.mm = mm;
    ka.mmLineOff = (int64_t)c0->mmLineOff();
    {  // multimem vector width: chunk starts (E*w) and tile offsets (T*w) 32-byte aligned
      const int64_t w = elemBytes(v[0]->dtype);
      bool a32 = (g.E * w) % 32 == 0 && (g.T * w) % 32 == 0 && ((uint64_t)g.n * w) % 32 == 0;
      for (auto* cl : v)
        a32 = a32 && ((uintptr_t)cl->buf[0] % 32 == 0) && ((uintptr_t)cl->buf[1] % 32 == 0);
      ka.mmVec32 = a32 ? 1 : 0;
    }
    int cta = 0;
    for (int i = 0; i < (int)v.size(); i++) {
      Call* cl = v[i];
      mscclProgram* p = cl->prog;
      r = checkDepth(cl->comm, p, g.I);
      if (r != mscclSuccess) return r;
      RankArgs& ra = ka.rank[i];
      ra.tbs = p->dTBs;
      ra.instrs = p->dInstr;
      ra.deps = p->dDeps;
      ra.sem = p->dSem;
      ra.gen = p->dSem + p->nTB;
      const int w = elemBytes(cl->dtype);
      size_t need = (size_t)p->algo.gpus[cl->comm->rank].sChunks * g.E * w;
      r = ensureScratch(cl->comm, p, need, cl->stream);
      if (r != mscclSuccess) return r;
      ra.buf[0] = cl->buf[0];
      ra.buf[1] = cl->buf[1];
      ra.buf[2] = p->dScratch;
      ra.nTB = p->nTB;
      ra.ctaStart = cta;
      ra.abortFlag = (uint32_t*)(cl->comm->region + cl->comm->abortOff());
      ra.hostAbort = cl->comm->hostAbortDev;
      ra.regMap = cl->comm->dRegMap;
      ra.peerRegion = cl->comm->dPeerRegion;
      ra.tbRec = p->dRec;
      ra.tbRecStride = p->dRec ? p->recStride : 0;
      ra.myRank = cl->comm->rank;
      ra.nRanks = cl->comm->nranks;
      if (mm) {  // NVSwitch multicast addresses of in / out (reading R23, hardware form)
        const int Rr = cl->comm->nranks;
        const size_t bytes[2] = {(size_t)g.n * blocksOf(p->algo.coll, BUF_IN, Rr) * w,
                                 (size_t)g.n * blocksOf(p->algo.coll, BUF_OUT, Rr) * w};
        for (int b = 0; b < 2; b++)
          for (auto& nv : cl->comm->nvls)
            if (ra.buf[b] >= nv.uc && ra.buf[b] + bytes[b] <= nv.uc + nv.size) ra.mcBuf[b] = nv.mc + (ra.buf[b] - nv.uc);
      }
      ra.stats = (unsigned long long*)(cl->comm->region + cl->comm->statsOff());
      ra.regMax = (int32_t)cl->comm->prm.regMax;
      if (direct == 1) {
        ra.directMask = 7;
      } else if ((direct == 2 || mm == 2) && !cl->aliased) {
        const int Rr = cl->comm->nranks;
        const size_t bytes[3] = {(size_t)g.n * blocksOf(p->algo.coll, BUF_IN, Rr) * w,
                                 (size_t)g.n * blocksOf(p->algo.coll, BUF_OUT, Rr) * w, need};
        for (int b = 0; b < 3; b++) {
          ra.bufRef[b] = bufferRef(cl->comm, ra.buf[b], bytes[b]);
          if (ra.bufRef[b] && direct == 2) ra.directMask |= 1 << b;
        }
      }
      if (mm == 2 && (!ra.bufRef[0] || !ra.bufRef[1]))
        return setErr(cl->comm, mscclInvalidUsage,
                      "a multimem program across processes needs sendbuff and recvbuff inside registered buffers "
                      "(mscclCommRegister; reading R23)");
      cta += p->nTB;
      if (cl->comm->sysScope || emulateCross) ka.sysScope = 1;
      if (direct == 1) cl->comm->launchesDirect1++;
      if (direct == 2 && ra.directMask) cl->comm->launchesDirect2++;
    }
    if (cta == 0) continue;
    auto pick = [&](bool wide) {
      return p0->hasMultimem ? (p0->hasReduce ? interpreterKernelMM(v[0]->dtype, v[0]->op)
                                              : copyKernelMM(elemBytes(v[0]->dtype)))
             : p0->hasReduce ? interpreterKernel(v[0]->dtype, v[0]->op, ka.proto, wide)
                             : copyKernel(elemBytes(v[0]->dtype), ka.proto, wide);
    };
    const void* fn = pick(false);
    int maxCta = 0;
    r = coResident(c0, fn, (int)c0->prm.threads, 0, maxCta);
    if (r != mscclSuccess) return r;
    if (cta > maxCta && ka.proto != 0 && !p0->hasMultimem) {
      // the LL / LL128 kernels run 1 CTA per SM (no spills); a larger launch takes their
      // 2-CTA/SM build instead
      fn = pick(true);
      r = coResident(c0, fn, (int)c0->prm.threads, 0, maxCta);
      if (r != mscclSuccess) return r;
    }
    if (cta > maxCta) {
      std::ostringstream o;
      o << "program needs " << cta << " co-resident CTAs on device " << c0->dev << " but at most " << maxCta
        << " fit (use fewer instances/channels, or fewer MSCCL_THREADS for more CTAs per SM)";
      return setErr(c0, mscclInvalidUsage, o.str());
    }
    DeviceGuard dg(c0->dev);
    void* args[] = {&ka};
    if (debugOn())
      fprintf(stderr, "[msccl] launch dev %d ranks %d program %s ctas %d threads %d n %lld E %lld T %lld I %d direct %d\n",
              c0->dev, ka.nLocal, p0->algo.name.c_str(), cta, (int)c0->prm.threads, (long long)g.n,
              (long long)g.E, (long long)g.T, g.I, direct);
    CUDACHECK(c0, cudaLaunchCooperativeKernel(fn, dim3(cta), dim3((unsigned)c0->prm.threads), args, 0,
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
  cl.aliased = false;
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
    cl.aliased = inplace;
    cl.buf[0] = (char*)sb;
    cl.buf[1] = rb;
  }
  cl.buf[2] = nullptr;
  return enqueue(cl);
}

}  // namespace

// ------------------------------------------------------------------ NVLS buffers (reading R23)
namespace {
template <typename F>
F driverFn(const char* name) {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &fn, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
    return nullptr;
  return (F)fn;
}
struct Drv {
  CUresult (*devAttr)(int*, CUdevice_attribute, CUdevice) = nullptr;
  CUresult (*mcCreate)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*) = nullptr;
  CUresult (*mcAddDevice)(CUmemGenericAllocationHandle, CUdevice) = nullptr;
  CUresult (*mcGran)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags) = nullptr;
  CUresult (*mcBindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                        unsigned long long) = nullptr;
  CUresult (*mcUnbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t) = nullptr;
  CUresult (*memCreate)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long) = nullptr;
  CUresult (*memRelease)(CUmemGenericAllocationHandle) = nullptr;
  CUresult (*memGran)(size_t*, const CUmemAllocationProp*, CUmemAllocationGranularity_flags) = nullptr;
  CUresult (*addrReserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long) = nullptr;
  CUresult (*addrFree)(CUdeviceptr, size_t) = nullptr;
  CUresult (*memMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long) = nullptr;
  CUresult (*memUnmap)(CUdeviceptr, size_t) = nullptr;
  CUresult (*setAccess)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t) = nullptr;
  bool ok = false;
};
const Drv& drv() {
  static Drv d;
  static bool init = false;
  if (!init) {
    init = true;
    d.devAttr = driverFn<decltype(d.devAttr)>("cuDeviceGetAttribute");
    d.mcCreate = driverFn<decltype(d.mcCreate)>("cuMulticastCreate");
    d.mcAddDevice = driverFn<decltype(d.mcAddDevice)>("cuMulticastAddDevice");
    d.mcGran = driverFn<decltype(d.mcGran)>("cuMulticastGetGranularity");
    d.mcBindMem = driverFn<decltype(d.mcBindMem)>("cuMulticastBindMem");
    d.mcUnbind = driverFn<decltype(d.mcUnbind)>("cuMulticastUnbind");
    d.memCreate = driverFn<decltype(d.memCreate)>("cuMemCreate");
    d.memRelease = driverFn<decltype(d.memRelease)>("cuMemRelease");
    d.memGran = driverFn<decltype(d.memGran)>("cuMemGetAllocationGranularity");
    d.addrReserve = driverFn<decltype(d.addrReserve)>("cuMemAddressReserve");
    d.addrFree = driverFn<decltype(d.addrFree)>("cuMemAddressFree");
    d.memMap = driverFn<decltype(d.memMap)>("cuMemMap");
    d.memUnmap = driverFn<decltype(d.memUnmap)>("cuMemUnmap");
    d.setAccess = driverFn<decltype(d.setAccess)>("cuMemSetAccess");
    d.ok = d.devAttr && d.mcCreate && d.mcAddDevice && d.mcGran && d.mcBindMem && d.mcUnbind && d.memCreate &&
           d.memRelease && d.memGran && d.addrReserve && d.addrFree && d.memMap && d.memUnmap && d.setAccess;
  }
  return d;
}
#define CUCHECK(c, call)                                                                   \
  do {                                                                                     \
    CUresult e_ = (call);                                                                  \
    if (e_ != CUDA_SUCCESS) {                                                              \
      std::ostringstream o_;                                                               \
      o_ << #call << " failed with CUresult " << (int)e_;                                  \
      return setErr((c), e_ == CUDA_ERROR_NOT_SUPPORTED ? mscclSystemError : mscclUnhandledCudaError, o_.str()); \
    }                                                                                      \
  } while (0)
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
  for (int i = 0; i < ndev; i++) {  // every rank of one device runs in one launch (MSCCL_MAX_LOCAL slots)
    int same = 0;
    for (int j = 0; j < ndev; j++) same += (devlist ? devlist[j] : j) == (devlist ? devlist[i] : i);
    if (same > MSCCL_MAX_LOCAL) {
      std::ostringstream o;
      o << "mscclCommInitAll: at most " << MSCCL_MAX_LOCAL << " ranks per device";
      return setErr(nullptr, mscclInvalidArgument, o.str());
    }
  }
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
    mscclResult_t ur = uploadPeerRegions(c);
    if (ur != mscclSuccess) return ur;
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
  if (nranks == 1) {
    c->connected = true;
    r = uploadPeerRegions(c);
    if (r != mscclSuccess) return r;
  }
  *comm = c;
  return mscclSuccess;
}

mscclResult_t mscclCommExportHandle(mscclComm_t c, void* handle, size_t* bytes) {
  if (!c || !handle) return setErr(c, mscclInvalidArgument, "null argument");
  memset(handle, 0, MSCCL_HANDLE_BYTES);
  DeviceGuard g(c->dev);
  cudaIpcMemHandle_t h;
  CUDACHECK(c, cudaIpcGetMemHandle(&h, c->region));
  memcpy(handle, &h, sizeof(h));
  // parameters that both ends of a connection must agree on (region layout, warp partition)
  // parameters both ends of a connection must agree on (region layout, slot geometry)
  // (MSCCL_DIRECT too: a receiver that publishes its destination expects the sender to store there)
  // word 1: MSCCL_DIRECT on/off | MSCCL_DIRECT_TILE << 1 (both must match: R15b, R19b)
  int64_t meta[8] = {(int64_t)c->regionBytes, (c->prm.direct != 0) | (c->prm.directTile << 1), c->prm.threads, c->prm.slots,
                     c->prm.slotBytes,         c->prm.llSlotBytes, c->prm.ll128SlotBytes, c->prm.maxChannels};
  static_assert(sizeof(cudaIpcMemHandle_t) + sizeof(meta) <= MSCCL_HANDLE_BYTES, "handle size");
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
    int64_t meta[8];
    memcpy(meta, h + sizeof(ih), sizeof(meta));
    const int64_t mine[8] = {(int64_t)c->regionBytes, (c->prm.direct != 0) | (c->prm.directTile << 1), c->prm.threads,
                             c->prm.slots,
                             c->prm.slotBytes,         c->prm.llSlotBytes, c->prm.ll128SlotBytes, c->prm.maxChannels};
    static const char* names[8] = {"region size", "MSCCL_DIRECT / MSCCL_DIRECT_TILE", "MSCCL_THREADS", "MSCCL_SLOTS", "MSCCL_SLOT_BYTES",
                                   "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES", "MSCCL_MAX_CHANNELS"};
    for (int k = 0; k < 8; k++)
      if (meta[k] != mine[k]) {
        std::ostringstream o;
        o << "rank " << p << " uses a different " << names[k] << " (" << meta[k] << " vs " << mine[k]
          << "): every rank must use the same MSCCL_* parameters";
        return setErr(c, mscclInvalidUsage, o.str());
      }
    void* ptr = nullptr;
    CUDACHECK(c, cudaIpcOpenMemHandle(&ptr, ih, cudaIpcMemLazyEnablePeerAccess));
    c->peerBase[p] = (char*)ptr;
    c->peerIpc[p] = true;
    c->sysScope = true;
  }
  c->connected = true;
  return uploadPeerRegions(c);
}

mscclResult_t mscclCommDestroy(mscclComm_t c) {
  if (!c) return mscclSuccess;
  {
    DeviceGuard g(c->dev);
    cudaDeviceSynchronize();
    for (auto* p : c->programs) freeProgram(p);
    c->programs.clear();
    for (auto* r : std::vector<mscclReg*>(c->regs))
      if (r) releaseReg(c, r);
    c->regs.clear();
    if (!c->nvls.empty()) {  // NVLS buffers the caller did not free (mscclNvlsFree of each rank)
      std::vector<void*> mine;
      for (auto& nv : c->nvls) mine.push_back(nv.uc);
      for (void* p : mine) mscclNvlsFree(&c, 1, &p);
    }
    cudaFree(c->dRegMap);
    cudaFree(c->dPeerRegion);
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

// ------------------------------------------------------------------ buffer registration (R15b)
namespace {
struct RegDesc {  // MSCCL_REG_DESC_BYTES bytes on the wire
  cudaIpcMemHandle_t h;
  uint64_t offset;  // registered range start - allocation base
  uint64_t size;
  int32_t idx, rank, single, pad;
};
static_assert(sizeof(RegDesc) <= MSCCL_REG_DESC_BYTES, "registration descriptor size");

typedef CUresult (*AddrRangeFn)(unsigned long long*, size_t*, unsigned long long);
}  // namespace

mscclResult_t mscclCommRegister(mscclComm_t c, void* buff, size_t size, mscclReg_t* out) {
  if (!c || !buff || !size || !out) return setErr(c, mscclInvalidArgument, "mscclCommRegister: null argument or size 0");
  int idx = -1;
  for (int i = 0; i < (int)c->prm.regMax && idx < 0; i++)
    if (i >= (int)c->regs.size() || !c->regs[i]) idx = i;
  if (idx < 0) return setErr(c, mscclInvalidArgument, "mscclCommRegister: MSCCL_MAX_REGISTRATIONS buffers already registered");
  // the allocation that holds [buff, buff+size) (CUDA IPC exports whole allocations)
  static AddrRangeFn addrRange = nullptr;
  if (!addrRange) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    CUDACHECK(c, cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q));
    if (!fn || q != cudaDriverEntryPointSuccess) return setErr(c, mscclSystemError, "cuMemGetAddressRange unavailable");
    addrRange = (AddrRangeFn)fn;
  }
  DeviceGuard g(c->dev);
  unsigned long long base = 0;
  size_t asize = 0;
  if (addrRange(&base, &asize, (unsigned long long)(uintptr_t)buff) != 0 ||
      (uintptr_t)buff + size > base + asize)
    return setErr(c, mscclInvalidArgument, "mscclCommRegister: range is not inside one device allocation");
  mscclReg* r = new mscclReg();
  r->comm = c;
  r->idx = idx;
  r->base = (char*)buff;
  r->size = size;
  r->allocBase = (char*)(uintptr_t)base;
  r->peerMapped.assign(c->nranks, nullptr);
  if ((int)c->regs.size() <= idx) c->regs.resize(idx + 1, nullptr);
  c->regs[idx] = r;
  *out = r;
  return mscclSuccess;
}

mscclResult_t mscclRegExport(mscclReg_t r, void* desc) {
  if (!r || !desc) return setErr(r ? r->comm : nullptr, mscclInvalidArgument, "mscclRegExport: null argument");
  mscclComm* c = r->comm;
  RegDesc d;
  memset(&d, 0, sizeof(d));
  d.offset = (uint64_t)(r->base - r->allocBase);
  d.size = r->size;
  d.idx = r->idx;
  d.rank = c->rank;
  d.single = c->clique ? 1 : 0;
  if (!c->clique) {
    DeviceGuard g(c->dev);
    CUDACHECK(c, cudaIpcGetMemHandle(&d.h, r->allocBase));
  }
  memset(desc, 0, MSCCL_REG_DESC_BYTES);
  memcpy(desc, &d, sizeof(d));
  return mscclSuccess;
}

mscclResult_t mscclRegConnect(mscclReg_t r, const void* all) {
  if (!r || !all) return setErr(r ? r->comm : nullptr, mscclInvalidArgument, "mscclRegConnect: null argument");
  mscclComm* c = r->comm;
  if (c->clique) {  // one address space: senders use raw pointers, nothing to map
    r->connected = true;
    return mscclSuccess;
  }
  DeviceGuard g(c->dev);
  for (int p = 0; p < c->nranks; p++) {
    if (p == c->rank) continue;
    RegDesc d;
    memcpy(&d, (const char*)all + (size_t)p * MSCCL_REG_DESC_BYTES, sizeof(d));
    if (d.rank != p || d.idx < 0 || d.idx >= c->prm.regMax || d.single)
      return setErr(c, mscclInvalidArgument, "mscclRegConnect: descriptors are not in rank order / from another kind of communicator");
    // one mapping per peer allocation (a handle can be opened once per process)
    std::string key(reinterpret_cast<const char*>(&d.h), sizeof(d.h));
    auto it = c->ipcCache.find({p, key});
    char* m = nullptr;
    if (it != c->ipcCache.end()) {
      m = it->second.first;
      it->second.second++;
    } else {
      void* ptr = nullptr;
      CUDACHECK(c, cudaIpcOpenMemHandle(&ptr, d.h, cudaIpcMemLazyEnablePeerAccess));
      m = (char*)ptr;
      c->ipcCache[{p, key}] = {m, 1};
    }
    r->peerMapped[p] = m;
    r->peerKeys.push_back({p, key});
    c->hRegMap[(size_t)p * c->prm.regMax + d.idx] = m + d.offset;
  }
  CUDACHECK(c, cudaMemcpy(c->dRegMap, c->hRegMap.data(), c->hRegMap.size() * sizeof(char*), cudaMemcpyHostToDevice));
  r->connected = true;
  return mscclSuccess;
}

mscclResult_t mscclCommDeregister(mscclComm_t c, mscclReg_t r) {
  if (!c || !r || r->comm != c) return setErr(c, mscclInvalidArgument, "mscclCommDeregister: bad arguments");
  DeviceGuard g(c->dev);
  CUDACHECK(c, cudaDeviceSynchronize());  // kernels that may still store into peers' mapped buffers
  releaseReg(c, r);
  return mscclSuccess;
}

// Direct-placement marking of the loader for one rank, for the oracle's race detector.
mscclResult_t mscclDebugDirectPlacement(const char* ir, size_t irBytes, int rank, int32_t* flags, int32_t* rdst,
                                        int maxInstr, int* nInstr) {
  if (!ir || !nInstr) return mscclInvalidArgument;
  try {
    Algo a = parseIR(ir, irBytes);
    Params prm = currentParams();
    validateIR(a, a.ngpus, (int)prm.slots, 1 << 15, 1 << 20);
    if (rank < 0 || rank >= a.ngpus) return mscclInvalidArgument;
    const DirectInfo di = directPlacement(a, rank);
    const GpuProgram& g = a.gpus[rank];
    int k = 0;
    for (size_t t = 0; t < g.tbs.size(); t++)
      for (size_t s = 0; s < g.tbs[t].steps.size(); s++, k++) {
        if (k >= maxInstr || !flags) continue;
        flags[k] = (di.sendDirect[t][s] ? 1 : 0) | (di.recvDirect[t][s] ? 2 : 0) | (di.recvPull[t][s] ? 4 : 0) |
                   (di.sendPulled[t][s] ? 8 : 0);
        if (rdst) {
          rdst[2 * k] = di.sendDirect[t][s] ? di.rdstBuf[t][s] : -1;
          rdst[2 * k + 1] = di.sendDirect[t][s] ? di.rdstOff[t][s] : -1;
        }
      }
    *nInstr = k;
  } catch (const IRError& e) {
    setErr(nullptr, mscclInvalidProgram, e.what());
    return mscclInvalidProgram;
  }
  return mscclSuccess;
}


mscclResult_t mscclNvlsSupported(int cudaDev, int* supported) {
  if (!supported) return mscclInvalidArgument;
  *supported = 0;
  const Drv& d = drv();
  if (!d.ok) return mscclSuccess;
  cudaFree(nullptr);  // a current context
  int v = 0;
  if (d.devAttr(&v, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, (CUdevice)cudaDev) == CUDA_SUCCESS) *supported = v;
  return mscclSuccess;
}

mscclResult_t mscclNvlsAlloc(mscclComm_t* comms, int n, size_t bytes, void** ptrs) {
  if (!comms || n < 1 || !bytes || !ptrs) return setErr(nullptr, mscclInvalidArgument, "mscclNvlsAlloc: bad arguments");
  mscclComm* c0 = comms[0];
  for (int i = 0; i < n; i++) {
    if (!comms[i] || comms[i]->rank != i || comms[i]->nranks != n || (n > 1 && comms[i]->clique != c0->clique) ||
        (n > 1 && !c0->clique))
      return setErr(comms[i], mscclInvalidArgument,
                    "mscclNvlsAlloc: pass every rank of one mscclCommInitAll communicator set, in rank order");
    for (int j = 0; j < i; j++)
      if (comms[j]->dev == comms[i]->dev)
        return setErr(comms[i], mscclInvalidUsage, "mscclNvlsAlloc: a multicast object binds one buffer per GPU "
                                                   "(virtual ranks cannot share one)");
  }
  const Drv& d = drv();
  if (!d.ok) return setErr(c0, mscclSystemError, "CUDA driver has no multicast API");
  for (int i = 0; i < n; i++) {
    int sup = 0;
    mscclNvlsSupported(comms[i]->dev, &sup);
    if (!sup) return setErr(comms[i], mscclSystemError, "device does not support NVSwitch multicast");
  }
  CUmulticastObjectProp mp;
  memset(&mp, 0, sizeof(mp));
  mp.numDevices = (unsigned)n;
  mp.size = bytes;
  mp.handleTypes = 0;
  size_t gran = 0, ugran = 0;
  {
    DeviceGuard g(c0->dev);
    cudaFree(nullptr);
    CUCHECK(c0, d.mcGran(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED));
  }
  CUmemAllocationProp ap;
  memset(&ap, 0, sizeof(ap));
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = c0->dev;
  CUCHECK(c0, d.memGran(&ugran, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
  size_t g2 = std::max(gran, ugran);
  mp.size = (bytes + g2 - 1) / g2 * g2;
  CUmemGenericAllocationHandle mc = 0;
  {
    DeviceGuard g(c0->dev);
    // the handle type only matters for export; some drivers refuse 0, so try the POSIX fd
    // type (the one NCCL uses for NVLS) first
    CUresult e = CUDA_ERROR_INVALID_VALUE;
    for (unsigned long long ht : {(unsigned long long)CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0ull,
                                  (unsigned long long)CU_MEM_HANDLE_TYPE_FABRIC}) {
      mp.handleTypes = ht;
      size_t gr = 0;
      if (d.mcGran(&gr, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS) continue;
      g2 = std::max(gr, ugran);
      mp.size = (bytes + g2 - 1) / g2 * g2;
      if ((e = d.mcCreate(&mc, &mp)) == CUDA_SUCCESS) break;
    }
    if (e != CUDA_SUCCESS) {
      std::ostringstream o;
      o << "cuMulticastCreate(numDevices=" << n << ", size=" << mp.size << ") failed with CUresult " << (int)e;
      return setErr(c0, e == CUDA_ERROR_NOT_SUPPORTED ? mscclSystemError : mscclUnhandledCudaError, o.str());
    }
  }
  const size_t size = mp.size;
  // everything created below is released again if a later step fails
  struct Made {
    int dev;
    CUmemGenericAllocationHandle phys;
    CUdeviceptr uc;
    bool bound, mapped;
  };
  std::vector<Made> made;
  CUdeviceptr mcva = 0;
  bool mcMapped = false;
  auto undo = [&]() {
    for (auto& m : made) {
      DeviceGuard g(m.dev);
      if (m.mapped) d.memUnmap(m.uc, size);
      if (m.uc) d.addrFree(m.uc, size);
      if (m.bound) d.mcUnbind(mc, (CUdevice)m.dev, 0, size);
      if (m.phys) d.memRelease(m.phys);
    }
    if (mcMapped) d.memUnmap(mcva, size);
    if (mcva) d.addrFree(mcva, size);
    d.memRelease(mc);
  };
#define NVTRY(c, call)                                                                        \
  do {                                                                                        \
    CUresult e_ = (call);                                                                     \
    if (e_ != CUDA_SUCCESS) {                                                                 \
      undo();                                                                                 \
      std::ostringstream o_;                                                                  \
      o_ << #call << " failed with CUresult " << (int)e_;                                     \
      return setErr((c), mscclUnhandledCudaError, o_.str());                                  \
    }                                                                                         \
  } while (0)
  for (int i = 0; i < n; i++) NVTRY(comms[i], d.mcAddDevice(mc, (CUdevice)comms[i]->dev));
  // the multicast address, mapped once and accessible from every device
  std::vector<CUmemAccessDesc> acc(n);
  for (int i = 0; i < n; i++) {
    acc[i].location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc[i].location.id = comms[i]->dev;
    acc[i].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  }
  for (int i = 0; i < n; i++) {
    DeviceGuard g(comms[i]->dev);
    cudaFree(nullptr);
    ap.location.id = comms[i]->dev;
    made.push_back({comms[i]->dev, 0, 0, false, false});
    Made& m = made.back();
    NVTRY(comms[i], d.memCreate(&m.phys, size, &ap, 0));
    NVTRY(comms[i], d.mcBindMem(mc, 0, m.phys, 0, size, 0));
    m.bound = true;
    NVTRY(comms[i], d.addrReserve(&m.uc, size, g2, 0, 0));
    NVTRY(comms[i], d.memMap(m.uc, size, 0, m.phys, 0));
    m.mapped = true;
    NVTRY(comms[i], d.setAccess(m.uc, size, acc.data(), acc.size()));  // peers reach it too (unicast form)
    if (i == 0) {
      NVTRY(comms[i], d.addrReserve(&mcva, size, g2, 0, 0));
      NVTRY(comms[i], d.memMap(mcva, size, 0, mc, 0));
      mcMapped = true;
      NVTRY(comms[i], d.setAccess(mcva, size, acc.data(), acc.size()));
    }
  }
#undef NVTRY
  for (int i = 0; i < n; i++) {
    mscclComm::Nvls nv{(char*)made[i].uc, (char*)mcva, size, (unsigned long long)made[i].phys,
                       (unsigned long long)mc, i == 0};
    comms[i]->nvls.push_back(nv);
    ptrs[i] = (void*)made[i].uc;
  }
  return mscclSuccess;
}

mscclResult_t mscclNvlsFree(mscclComm_t* comms, int n, void** ptrs) {
  if (!comms || n < 1 || !ptrs) return mscclInvalidArgument;
  const Drv& d = drv();
  std::vector<mscclComm::Nvls> owners;
  for (int i = 0; i < n; i++) {  // every rank's memory first ...
    mscclComm* c = comms[i];
    DeviceGuard g(c->dev);
    CUDACHECK(c, cudaDeviceSynchronize());
    auto it = std::find_if(c->nvls.begin(), c->nvls.end(), [&](const mscclComm::Nvls& x) { return x.uc == ptrs[i]; });
    if (it == c->nvls.end()) return setErr(c, mscclInvalidArgument, "mscclNvlsFree: not an NVLS buffer of this rank");
    d.memUnmap((CUdeviceptr)it->uc, it->size);
    d.addrFree((CUdeviceptr)it->uc, it->size);
    d.mcUnbind((CUmemGenericAllocationHandle)it->mcHandle, (CUdevice)c->dev, 0, it->size);
    d.memRelease((CUmemGenericAllocationHandle)it->phys);
    if (it->owner) owners.push_back(*it);
    c->nvls.erase(it);
  }
  for (auto& o : owners) {  // ... then the multicast address and object
    d.memUnmap((CUdeviceptr)o.mc, o.size);
    d.addrFree((CUdeviceptr)o.mc, o.size);
    d.memRelease((CUmemGenericAllocationHandle)o.mcHandle);
  }
  return mscclSuccess;
}

mscclResult_t mscclCommGetStats(mscclComm_t c, int64_t* stats, int n) {
  if (!c || !stats || n < 1) return mscclInvalidArgument;
  DeviceGuard g(c->dev);
  uint64_t dev[2] = {0, 0};
  CUDACHECK(c, cudaMemcpy(dev, c->region + c->statsOff(), sizeof(dev), cudaMemcpyDeviceToHost));
  const int64_t v[5] = {(int64_t)dev[0], (int64_t)c->launchesDirect1, (int64_t)c->launchesDirect2, (int64_t)dev[1],
                        (int64_t)c->depthChecks};
  for (int i = 0; i < n && i < 5; i++) stats[i] = v[i];
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
  p->hasMultimem = p->algo.hasMultimem();
  for (auto& tb : g.tbs)
    for (auto& in : tb.steps)
      if (in.op == OP_RCS || in.op == OP_RRS || in.op == OP_RRCS) p->forwards = true;
  if (p->hasMultimem && c->nranks > MSCCL_MM_MAX_RANKS)
    return setErr(c, mscclInvalidProgram, "V11: multimem programs support at most 16 ranks");
  const uint32_t tag = ++c->loadCounter;
  const DirectInfo dinfo = directPlacement(p->algo, c->rank);
  std::vector<DevTB> tbs(p->nTB);
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
    d.mmId = -1;
    d.mmTag = tag;
    for (auto& in : tb.steps)
      if (isMultimem(in.op)) d.mmId = tb.id;
    if (d.mmId >= MSCCL_MM_MAX_TB)
      return setErr(c, mscclInvalidProgram, "V11: a multimem thread block id must be < 64 (group-barrier lines)");
    const int pr = p->algo.proto;
    if (tb.send >= 0) {
      d.sendFifo = c->peerBase[tb.send] + c->fifoOff(pr, c->rank, tb.chan);
      d.sendHead = (uint64_t*)(c->peerBase[tb.send] + c->flagOff(0, c->rank, tb.chan));
      d.sendAck = (uint64_t*)(c->region + c->flagOff(1, tb.send, tb.chan));
      d.sendCnt = (uint64_t*)(c->region + c->flagOff(2, tb.send, tb.chan));
      d.sendReady = (uint64_t*)(c->region + c->flagOff(4, tb.send, tb.chan));
    }
    if (tb.recv >= 0) {
      d.recvFifo = c->region + c->fifoOff(pr, tb.recv, tb.chan);
      d.recvHead = (uint64_t*)(c->region + c->flagOff(0, tb.recv, tb.chan));
      d.recvAck = (uint64_t*)(c->peerBase[tb.recv] + c->flagOff(1, c->rank, tb.chan));
      d.recvCnt = (uint64_t*)(c->region + c->flagOff(3, tb.recv, tb.chan));
      d.recvReady = (uint64_t*)(c->peerBase[tb.recv] + c->flagOff(4, c->rank, tb.chan));
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
      if (dinfo.recvPull[t][si]) {  // reading R30
        di.flags |= DI_RECV_PULL;
        di.chainLen = (uint16_t)tb.recv;
        di.pullOff = (uint32_t)dinfo.pullOff[t][si];
      }
      if (dinfo.sendPulled[t][si]) di.flags |= DI_SEND_PULLED;
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
  // per-block records for the latency kernels: DevTB followed by its instructions, fixed
  // stride, so one round trip stages both (only when every list fits the shared stage)
  {
    int maxSteps = 0;
    for (auto& d : tbs) maxSteps = std::max(maxSteps, d.nSteps);
    if (p->nTB && maxSteps <= 64) {
      p->recStride = (int64_t)(sizeof(DevTB) + (size_t)maxSteps * sizeof(DevInstr) + 15) / 16 * 16;
      std::vector<char> host((size_t)p->nTB * p->recStride, 0);
      for (int t = 0; t < p->nTB; t++) {
        memcpy(host.data() + (size_t)t * p->recStride, &tbs[t], sizeof(DevTB));
        if (tbs[t].nSteps)
          memcpy(host.data() + (size_t)t * p->recStride + sizeof(DevTB), &ins[tbs[t].instrStart],
                 (size_t)tbs[t].nSteps * sizeof(DevInstr));
      }
      CUDACHECK(c, cudaMalloc(&p->dRec, host.size()));
      CUDACHECK(c, cudaMemcpy(p->dRec, host.data(), host.size(), cudaMemcpyHostToDevice));
    }
  }
  // scratch pre-sized for the largest call of the size range: every chunk of a
  // call with count*w < maxBytes has E*w <= maxBytes/cb + 16 bytes (reading R1)
  if (maxBytes > 0 && g.sChunks > 0) {
    const int cb = std::max(1, p->algo.gpus[0].iChunks / blocksOf(p->algo.coll, BUF_IN, p->algo.ngpus));
    const size_t perChunk = maxBytes / cb + 32;
    p->scratchBytes = ((size_t)g.sChunks * perChunk + 4095) / 4096 * 4096;
    CUDACHECK(c, cudaMalloc(&p->dScratch, p->scratchBytes));
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

mscclResult_t mscclDebugSetGeneration(mscclProgram_t p, uint64_t generation) {
  if (!p) return mscclInvalidArgument;
  if (!p->nTB) return mscclSuccess;
  DeviceGuard dg(p->comm->dev);
  std::vector<uint64_t> g(p->nTB, generation);
  CUDACHECK(p->comm, cudaDeviceSynchronize());
  CUDACHECK(p->comm, cudaMemcpy(p->dSem + p->nTB, g.data(), g.size() * sizeof(uint64_t), cudaMemcpyHostToDevice));
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
      if (direct == 1 && (p->comm->prm.directHints & 16) && di.sendPulled[t][s]) c = 0;  // reading R30
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
