// Structures shared by the host runtime and the interpreter kernel.
//
// Instruction record = Fig. 5 lines 1-5: opcode, src/dst buffer + chunk
// offset, count, dependency list (depBid/depStep generalised to a variable-length table,
// DESIGN.md reading R4) and hasDep.
#pragma once
#include <stdint.h>

namespace msccl {

#define MSCCL_MAX_LOCAL 16  // ranks that one kernel launch may cover (virtual ranks)
#define MSCCL_FLAG_WORDS 16 // u64 flag words per connection counter: one per warp (<= 512 threads)
#define MSCCL_CTA_MAP 512   // largest grid whose CTA -> (rank, thread block) order the host sets

// DI_SEND_TERMINAL: a direct send whose receiving instruction is a plain recv (the data is
// not forwarded by the receiver's thread block: a cache hint only)
enum { DI_SEND_DIRECT = 1, DI_RECV_DIRECT = 2, DI_CHAIN_HEAD = 4, DI_SEND_TERMINAL = 8 };

struct DevInstr {     // 32 bytes
  uint8_t op, srcBuf, dstBuf, nDeps;
  uint16_t cnt, hasDep;
  uint32_t srcOff, dstOff, depStart;
  // direct placement (reading R15): the message lands in the receiver's destination chunk
  // instead of its FIFO slot. flags: DI_SEND_DIRECT (this send writes peer rdstBuf/rdstOff),
  // DI_RECV_DIRECT (the data of this receive is already in dst when its head arrives).
  uint8_t flags, rdstBuf;
  uint16_t chainLen;          // DI_CHAIN_HEAD: this and the next chainLen-1 local ops fold into one pass
  uint32_t rdstOff, pad1;
};

// One thread block of one rank (= one CTA). Connection pointers are resolved at load time
// from the communicator's peer mapping (receiver-side FIFOs, §6.1).
struct DevTB {
  int32_t nSteps;
  uint32_t instrStart;
  int32_t tbId;
  int32_t sendPeer;           // rank of the send peer (-1 if none)
  // send connection (peer = receiver): FIFO and head counter live in the PEER's region.
  // head/ack are arrays of MSCCL_FLAG_WORDS words: with warp flags (Simple protocol) warp w
  // of the sender and warp w of the receiver own word w (reading R18); block-level protocols
  // wait on word 0 and post every word.
  char* sendFifo;             // peer FIFO base for (me -> peer, chan); nullptr if no send peer
  uint64_t* sendHead;         // peer: messages posted by me
  uint64_t* sendAck;          // mine: messages the peer consumed (written by the peer)
  uint64_t* sendCnt;          // mine: persistent count of messages I posted
  // receive connection (peer = sender)
  char* recvFifo;             // my FIFO base for (peer -> me, chan)
  uint64_t* recvHead;         // mine: messages the peer posted (written by the peer)
  uint64_t* recvAck;          // peer: messages I consumed
  uint64_t* recvCnt;          // mine: persistent count of messages I consumed
};

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
  int32_t useTma;             // Simple protocol: bulk-copy (TMA) pipeline through shared memory
  int32_t direct;             // honour DI_*_DIRECT flags (all ranks in this launch, rank == slot)
  int32_t warpFlags;          // Simple protocol: per-warp head/ack flags, no block barrier per message (R18)
  int32_t prefetch;           // Simple protocol: bulk L2 prefetch of the local operand before a receive wait
  int32_t directHints;        // bit 0: terminal direct sends store L2 evict_first; bit 1: a direct
                              // forward demotes the lines it read to evict_normal (cache hints)
  uint64_t timeoutNs;
  uint64_t* trace;            // MSCCL_TRACE builds: per-CTA phase times (ns), else null
  // CTA c runs thread block ctaMap[c] & 4095 of local rank ctaMap[c] >> 12 (work-balanced
  // placement: the thread blocks that move the most bytes get the lowest block indices, which
  // the hardware spreads over distinct SMs first); ctaMapN == 0: rank by prefix sums
  int32_t ctaMapN;
  uint16_t ctaMap[MSCCL_CTA_MAP];
};
static_assert(sizeof(KernelArgs) <= 4096, "kernel parameter space");

}  // namespace msccl
