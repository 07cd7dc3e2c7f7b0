// Host-side MSCCL-IR model, parser and validator (product side; independent of oracle/).
//
// MSCCL-IR: program -> GPU programs -> thread blocks {send peer, recv peer, channel} ->
// ordered instructions {op, src buf/chunk, dst buf/chunk, count, deps, hasDep}
// (MSCCLang §5, Fig. 4, Fig. 5).
#pragma once
#include <stdexcept>
#include <string>
#include <utility>
#include <vector>

namespace msccl {

enum Coll { COLL_ALLREDUCE = 0, COLL_ALLGATHER = 1, COLL_REDUCESCATTER = 2, COLL_ALLTOALL = 3, COLL_CUSTOM = 4 };
enum Proto { PROTO_SIMPLE = 0, PROTO_LL = 1, PROTO_LL128 = 2 };

// opcodes (also the device encoding)
enum OpCode { OP_NOP = 0, OP_SEND = 1, OP_RECV = 2, OP_COPY = 3, OP_REDUCE = 4, OP_RRC = 5, OP_RRS = 6,
              OP_RRCS = 7, OP_RCS = 8,
              // multimem (NVLS) ops, reading R23: the same chunk on every rank of the group
              OP_MRD = 9,    // dst_q <- (+)_p src_p                 (multimem.ld_reduce)
              OP_MST = 10,   // dst_p <- src_q for every rank p      (multimem.st)
              OP_MRS = 11,   // v = (+)_p src_p; dst_p <- v           (ld_reduce + st)
              OP_COUNT = 12 };
inline bool isMultimem(int op) { return op == OP_MRD || op == OP_MST || op == OP_MRS; }
enum BufId { BUF_IN = 0, BUF_OUT = 1, BUF_SC = 2, BUF_NONE = 3 };

// per-op roles (§4.2): receives, sends, reads src, writes dst
struct OpRole { bool recv, send, src, dst; };
inline OpRole opRole(int op) {
  static const OpRole t[OP_COUNT] = {
      {false, false, false, false},  // nop
      {false, true, true, false},    // send
      {true, false, false, true},    // recv
      {false, false, true, true},    // copy
      {false, false, true, true},    // reduce (also reads dst)
      {true, false, true, true},     // rrc
      {true, true, true, false},     // rrs
      {true, true, true, true},      // rrcs
      {true, true, false, true},     // rcs
      {false, false, true, true},    // mrd
      {false, false, true, true},    // mst
      {false, false, true, true},    // mrs
  };
  return t[op];
}

struct IRError : std::runtime_error {
  explicit IRError(const std::string& s) : std::runtime_error(s) {}
};

struct Instr {
  int op = OP_NOP, srcBuf = BUF_NONE, srcOff = -1, dstBuf = BUF_NONE, dstOff = -1, cnt = 1;
  std::vector<std::pair<int, int>> deps;  // (tb, step)
  bool hasDep = false;
};

struct ThreadBlock {
  int id = 0, send = -1, recv = -1, chan = 0;
  std::vector<Instr> steps;
};

struct GpuProgram {
  int id = 0, iChunks = 0, oChunks = 0, sChunks = 0;
  std::vector<ThreadBlock> tbs;
};

struct Algo {
  std::string name;
  int coll = COLL_ALLREDUCE, ngpus = 0, proto = PROTO_SIMPLE, nchannels = 1;
  bool inplace = false, aliassafe = false;
  std::vector<GpuProgram> gpus;
  int maxCnt() const;
  bool hasReduce() const;
  bool hasMultimem() const;
};

Algo parseIR(const char* text, size_t len);  // throws IRError (rule V1)

// Throws IRError("Vn: ...") on the first violated rule (V1..V9).
void validateIR(Algo& a, int nranks, int slots, int maxTbs, int maxChannels, int iters = 2);
// V9 alone at a given pipeline depth (the launch's real I); throws IRError("V9: ...").
void deadlockCheckIR(const Algo& a, int slots, int iters);

// Direct placement analysis (reading R15). For rank `rank`: recvDirect[tb][step] = the
// receive may find its data already in its destination (op r / rcs whose destination
// chunks no other instruction of the rank touches unless ordered after it);
// sendDirect[tb][step] = the matching receive on the peer is direct (+ its dst buf/off).
// recvPull[tb][step] = the receive may read its message from the sender's input chunk
// pullOff (reading R30); sendPulled[tb][step] = the matching receive on the peer pulls.
struct DirectInfo {
  std::vector<std::vector<char>> recvDirect, sendDirect, recvPull, sendPulled;
  std::vector<std::vector<int>> rdstBuf, rdstOff, rterminal, pullOff;
};
DirectInfo directPlacement(const Algo& a, int rank);

// blocks per buffer for a collective (reading R1)
int blocksOf(int coll, int buf, int R);

}  // namespace msccl
