// Structures shared by the host runtime and the interpreter kernel.
//
// Instruction record = Fig. 5 lines 1-5: opcode, src/dst buffer + chunk
// offset, count, dependency list (depBid/depStep generalised to a variable-length table,
// DESIGN.md reading R4) and hasDep.
#pragma once
#include <stdint.h>

namespace msccl {

#ifndef MSCCL_MAX_LOCAL
#define MSCCL_MAX_LOCAL 8    // ranks that one kernel launch may cover (virtual ranks); every RankArgs slot
                             // is a kernel parameter: 16 -> 8 cut the launch floor by ~0.4 us
#endif
#define MSCCL_FLAG_STRIDE 16 // u64 words between connection counters (one 128-byte line each)
#define MSCCL_REF_REG (1ull << 63)  // destination reference: registered-buffer (index, offset) form
#define MSCCL_MM_MAX_TB 64   // thread-block ids that may hold multimem ops (group-barrier lines)
#define MSCCL_MM_MAX_RANKS 16
#ifndef MSCCL_MAX_THREADS
#define MSCCL_MAX_THREADS 256  // threads per CTA (MSCCL_THREADS <= this); 2 CTAs per SM at 256
#endif

// DI_SEND_TERMINAL: a direct send whose receiving instruction is a plain recv (the data is
// not forwarded by the receiver's thread block: a cache hint only)
// DI_RECV_PULL / DI_SEND_PULLED (reading R30): with every rank in the launch (direct == 1) and
// MSCCL_DIRECT_HINTS bit 4, the receive reads its message from the sender's input chunk pullOff
// (rank chainLen) and the send moves no data (it still posts its head flag).
enum { DI_SEND_DIRECT = 1, DI_RECV_DIRECT = 2, DI_CHAIN_HEAD = 4, DI_SEND_TERMINAL = 8, DI_RECV_PULL = 16,
       DI_SEND_PULLED = 32 };

struct DevInstr {     // 32 bytes
  uint8_t op, srcBuf, dstBuf, nDeps;
  uint16_t cnt, hasDep;
  uint32_t srcOff, dstOff, depStart;
  // direct placement (reading R15): the message lands in the receiver's destination chunk
  // instead of its FIFO slot. flags: DI_SEND_DIRECT (this send writes peer rdstBuf/rdstOff),
  // DI_RECV_DIRECT (the data of this receive is already in dst when its head arrives).
  uint8_t flags, rdstBuf;
  uint16_t chainLen;          // DI_CHAIN_HEAD: this and the next chainLen-1 local ops fold into one pass;
                              // DI_RECV_PULL: the sender's rank
  uint32_t rdstOff, pullOff;  // pullOff: DI_RECV_PULL: the sender's input chunk
};

// One thread block of one rank (= one CTA). Connection pointers are resolved at load time
// from the communicator's peer mapping (receiver-side FIFOs, §6.1).
struct DevTB {
  int32_t nSteps;
  uint32_t instrStart;
  int32_t tbId;
  int32_t sendPeer;           // rank of the send peer (-1 if none)
  // send connection (peer = receiver): FIFO and head counter live in the PEER's region; the
  // FIFO is the region of this program's protocol (each protocol has its own slots).
  char* sendFifo;             // peer FIFO base for (me -> peer, chan); nullptr if no send peer
  uint64_t* sendHead;         // peer: messages posted by me
  uint64_t* sendAck;          // mine: messages the peer consumed (written by the peer)
  uint64_t* sendCnt;          // mine: [0] messages I posted, [1] launches on this connection
  uint64_t* sendReady;        // mine: [0] receiver's launch ordinal, [1..3] its in/out/sc refs, [4] its tile T
  // receive connection (peer = sender)
  char* recvFifo;             // my FIFO base for (peer -> me, chan)
  uint64_t* recvHead;         // mine: messages the peer posted (written by the peer)
  uint64_t* recvAck;          // peer: messages I consumed
  uint64_t* recvCnt;          // mine: [0] messages I consumed, [1] launches on this connection
  uint64_t* recvReady;        // peer: the sender's ready line for this connection (I write it)
  int32_t mmId;               // multimem thread block: its group-barrier line index (tb id), else -1
  uint32_t mmTag;             // the program's load ordinal on this communicator (group-barrier epoch)
  int32_t pad[2];
};
static_assert(sizeof(DevTB) % 16 == 0, "DevTB is staged with 16-byte loads");

struct RankArgs {
  const DevTB* tbs;
  const DevInstr* instrs;
  const uint64_t* deps;       // (tb << 48) | (step << 32) | nSteps of tb (DevTB::depWord)
  uint64_t* sem;              // per-TB semaphores (monotone, reading R4)
  uint64_t* gen;              // per-TB launch generation
  char* buf[3];               // in, out, scratch base pointers for this call
  int32_t nTB;
  int32_t ctaStart;           // first CTA of this rank in the grid
  uint32_t* abortFlag;        // this rank's abort word (device memory of its region)
  uint32_t* hostAbort;        // this rank's host-mapped pinned word (watchdog report)
  // cross-launch direct placement (reading R15b): how a sender reaches this rank's in/out/sc
  // in this call (raw pointer, MSCCL_REF_REG|idx<<40|offset, or 0 = not reachable), the mask of
  // buffers whose direct receives are honoured, and this rank's table of peers' registered
  // buffers mapped into this process: regMap[peer * regMax + idx]
  uint64_t bufRef[3];
  char* const* regMap;
  int32_t regMax;
  int32_t directMask;
  unsigned long long* stats;  // this rank's counters (region): [0] cross-launch handshakes that
                              // resolved a direct destination (mscclCommGetStats)
  char* const* peerRegion;    // every rank's shared region in this address space (group barriers)
  int32_t myRank, nRanks;
  // latency kernels: each thread block's DevTB followed by its instructions, one record per
  // block at tbRec + tb * tbRecStride (0 = no records: instructions longer than the stage)
  const char* tbRec;
  int64_t tbRecStride;
  // NVSwitch multicast addresses of this rank's in / out buffers when they lie inside an
  // NVLS buffer (mscclNvlsAlloc), else null: multimem ops on them use multimem.ld_reduce /
  // multimem.st (the hardware form of reading R23)
  char* mcBuf[2];
};

struct KernelArgs {
  RankArgs rank[MSCCL_MAX_LOCAL];
  int32_t nLocal;
  int32_t I;                  // pipeline iterations (reading R3)
  int64_t n;                  // elements per block
  int64_t E;                  // elements per chunk
  int64_t T;                  // tile elements
  int32_t cb;                 // chunks per block
  int32_t blocks[3];          // blocks of in / out / scratch (scratch: 1)
  int32_t slots;              // FIFO slots per connection
  int32_t proto;              // 0 Simple, 1 LL
  int64_t slotBytes;
  int32_t sysScope;           // 1 when any peer is another GPU
  // direct placement (reading R15): 0 off; 1 every rank is in this launch (rank == slot);
  // 2 cross-launch (ranks in other launches / processes, ready handshake per connection)
  int32_t direct;
  int32_t directHints;        // L2 hints (interp.cuh HINT_*): bit 0 terminal direct sends evict_first,
                              // bit 1 demote read forwarded lines, bit 2 FIFO stores / bit 3 direct
                              // forwards evict_normal; bit 4 pulled first hops with direct == 1
                              // (reading R30) (default 25 = bits 0, 3, 4)
  // multimem ops (reading R23): 0 none; 1 every rank in this launch (slot r = rank r, buffers
  // from the launch arguments, no barrier); 2 cross-launch (group barrier lines publish the
  // ranks' buffer references at the start and completion at the end)
  int32_t mm;
  int32_t mmVec32;            // multimem: every chunk / tile span is 32-byte aligned (32-byte vectors)
  int32_t tileIsChunk;        // reading R19: T = E, every message a direct placement (no FIFO slot)
  int64_t mmLineOff;          // offset of the group-barrier lines in every region
  uint64_t timeoutNs;         // device watchdog; 0 = disabled
  uint64_t* trace;            // MSCCL_TRACE builds: per-CTA phase times (ns), else null
};
static_assert(sizeof(KernelArgs) <= 4096, "kernel parameter space");
static_assert(sizeof(KernelArgs) % 4 == 0, "KernelArgs is staged as 32-bit words");

}  // namespace msccl
