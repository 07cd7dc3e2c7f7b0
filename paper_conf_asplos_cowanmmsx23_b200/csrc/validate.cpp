// MSCCL-IR validator (DESIGN.md rules V2..V9). Runs on the host at mscclLoadProgram.
//
// V9 is an abstract execution of the program with counters only: each thread block walks
// its instruction list once per pipeline iteration; a receive needs a posted message on
// its connection, a send needs a free FIFO slot (at most `slots` outstanding, §6.1
// P:L1313-1322), a dependency needs the named step done in the same iteration (Fig. 5
// P:L1294-1307). No progress in a full sweep before completion = deadlock.
#include <algorithm>
#include <map>
#include <sstream>
#include <tuple>

#include "ir.h"

namespace msccl {

int blocksOf(int coll, int buf, int R) {
  if (buf == BUF_IN) return (coll == COLL_REDUCESCATTER || coll == COLL_ALLTOALL) ? R : 1;
  if (buf == BUF_OUT) return (coll == COLL_ALLGATHER || coll == COLL_ALLTOALL) ? R : 1;
  return 1;
}

namespace {

[[noreturn]] void fail(const char* rule, const std::string& msg) { throw IRError(std::string(rule) + ": " + msg); }

std::string where(int g, int tb, int s = -1) {
  std::ostringstream o;
  o << "rank " << g << " tb " << tb;
  if (s >= 0) o << " step " << s;
  return o.str();
}

typedef std::tuple<int, int, int> ConnKey;  // (src, dst, chan)

void deadlockCheck(const Algo& a, int slots, int iters) {
  struct TBRef { int g, tb; long long done, total; };
  std::vector<TBRef> tbs;
  std::map<ConnKey, long long> posted, consumed;
  for (auto& g : a.gpus)
    for (auto& tb : g.tbs) tbs.push_back({g.id, tb.id, 0, (long long)tb.steps.size() * iters});
  std::map<std::pair<int, int>, long long*> prog;
  for (auto& r : tbs) prog[{r.g, r.tb}] = &r.done;
  for (;;) {
    bool progressed = false, finished = true;
    for (auto& r : tbs) {
      const ThreadBlock& tb = a.gpus[r.g].tbs[r.tb];
      long long n = (long long)tb.steps.size();
      while (r.done < r.total) {
        long long t = r.done / n;
        const Instr& in = tb.steps[r.done % n];
        OpRole ro = opRole(in.op);
        bool ok = true;
        for (auto& d : in.deps) {
          long long dn = (long long)a.gpus[r.g].tbs[d.first].steps.size();
          if (*prog[{r.g, d.first}] < t * dn + d.second + 1) { ok = false; break; }
        }
        ConnKey rk(tb.recv, r.g, tb.chan), sk(r.g, tb.send, tb.chan);
        if (ok && ro.recv && posted[rk] <= consumed[rk]) ok = false;
        if (ok && ro.send && posted[sk] - consumed[sk] >= slots) ok = false;
        if (!ok) break;
        if (ro.recv) consumed[rk]++;
        if (ro.send) posted[sk]++;
        r.done++;
        progressed = true;
      }
      if (r.done < r.total) finished = false;
    }
    if (finished) return;
    if (!progressed) {
      std::ostringstream o;
      o << "deadlock with " << slots << " FIFO slots:";
      int shown = 0;
      for (auto& r : tbs)
        if (r.done < r.total && shown++ < 6) {
          long long n = (long long)a.gpus[r.g].tbs[r.tb].steps.size();
          o << " [" << where(r.g, r.tb, (int)(r.done % n)) << " iteration " << r.done / n << "]";
        }
      fail("V9", o.str());
    }
  }
}

}  // namespace

void deadlockCheckIR(const Algo& a, int slots, int iters) { deadlockCheck(a, slots, iters); }

void validateIR(Algo& a, int nranks, int slots, int maxTbs, int maxChannels, int iters) {
  const int R = a.ngpus;
  if (nranks > 0 && R != nranks) {
    std::ostringstream o;
    o << "program is for " << R << " ranks, communicator has " << nranks;
    fail("V2", o.str());
  }
  if ((int)a.gpus.size() != R) fail("V2", "number of <gpu> elements differs from ngpus");
  std::sort(a.gpus.begin(), a.gpus.end(), [](const GpuProgram& x, const GpuProgram& y) { return x.id < y.id; });
  for (int i = 0; i < R; i++)
    if (a.gpus[i].id != i) fail("V2", "gpu ids must be 0..ngpus-1");
  const GpuProgram& g0 = a.gpus[0];
  for (auto& g : a.gpus)
    if (g.iChunks != g0.iChunks || g.oChunks != g0.oChunks) fail("V3", where(g.id, 0) + ": chunk counts differ from rank 0");
  int ci = g0.iChunks, co = g0.oChunks;
  bool ok = false;
  switch (a.coll) {
    case COLL_ALLREDUCE: ok = ci == co && ci >= 1; break;
    case COLL_ALLGATHER: ok = co == R * ci && ci >= 1; break;
    case COLL_REDUCESCATTER: ok = ci == R * co && co >= 1; break;
    case COLL_ALLTOALL: ok = ci == co && ci >= R && ci % R == 0; break;
    case COLL_CUSTOM: ok = ci == co && ci >= 1; break;
  }
  if (!ok) fail("V3", "chunk counts do not fit the collective");
  if (a.inplace && a.coll != COLL_ALLREDUCE && a.coll != COLL_CUSTOM) fail("V3", "in-place programs are only defined for allreduce/custom");

  std::map<ConnKey, std::pair<int, int>> senders, receivers;  // -> (gpu, tb)
  for (auto& g : a.gpus) {
    if ((int)g.tbs.size() > maxTbs) {
      std::ostringstream o;
      o << "rank " << g.id << " has " << g.tbs.size() << " thread blocks > " << maxTbs;
      fail("V4", o.str());
    }
    std::sort(g.tbs.begin(), g.tbs.end(), [](const ThreadBlock& x, const ThreadBlock& y) { return x.id < y.id; });
    for (size_t i = 0; i < g.tbs.size(); i++)
      if (g.tbs[i].id != (int)i) fail("V1", where(g.id, (int)i) + ": thread block ids must be 0..n-1");
    int nch[3] = {g.iChunks, g.oChunks, g.sChunks};
    if (a.inplace) nch[BUF_OUT] = g.iChunks;
    for (auto& tb : g.tbs) {
      for (int p : {tb.send, tb.recv})
        if (p != -1 && (p < 0 || p >= R || p == g.id)) fail("V4", where(g.id, tb.id) + ": bad peer");
      if (tb.chan < 0 || tb.chan >= maxChannels) fail("V4", where(g.id, tb.id) + ": channel out of range");
      if (tb.send >= 0) {
        ConnKey k(g.id, tb.send, tb.chan);
        if (senders.count(k)) fail("V5", where(g.id, tb.id) + ": connection has two sending thread blocks");
        senders[k] = {g.id, tb.id};
      }
      if (tb.recv >= 0) {
        ConnKey k(tb.recv, g.id, tb.chan);
        if (receivers.count(k)) fail("V5", where(g.id, tb.id) + ": connection has two receiving thread blocks");
        receivers[k] = {g.id, tb.id};
      }
      for (size_t s = 0; s < tb.steps.size(); s++) {
        const Instr& in = tb.steps[s];
        std::string w = where(g.id, tb.id, (int)s);
        OpRole ro = opRole(in.op);
        if (ro.send && tb.send < 0) fail("V6", w + ": instruction sends but the thread block has no send peer");
        if (ro.recv && tb.recv < 0) fail("V6", w + ": instruction receives but the thread block has no receive peer");
        if (in.op != OP_NOP && (in.cnt < 1 || in.cnt > 65535)) fail("V6", w + ": cnt out of range");
        struct { bool used; int buf, off; } acc[2] = {{ro.src, in.srcBuf, in.srcOff}, {ro.dst, in.dstBuf, in.dstOff}};
        for (auto& x : acc) {
          if (!x.used) continue;
          if (x.buf == BUF_NONE) fail("V6", w + ": missing buffer");
          if (x.off < 0 || (long long)x.off + in.cnt > nch[x.buf]) fail("V6", w + ": chunk range exceeds the buffer");
        }
        if (ro.dst && in.dstBuf == BUF_IN && !a.inplace) fail("V3", w + ": out-of-place program writes the input buffer");
        if (isMultimem(in.op) && (in.srcBuf == BUF_SC || in.dstBuf == BUF_SC))
          fail("V11", w + ": multimem op on the scratch buffer (per-rank sizes)");
        for (auto& d : in.deps) {
          if (d.first == tb.id) fail("V8", w + ": depends on its own thread block");
          if (d.first < 0 || d.first >= (int)g.tbs.size() || d.second < 0 ||
              d.second >= (int)g.tbs[d.first].steps.size())
            fail("V8", w + ": dependency names a missing step");
          if (!g.tbs[d.first].steps[d.second].hasDep) fail("V8", w + ": dependency target does not set hasdep");
        }
      }
    }
  }
  for (auto& kv : senders)
    if (!receivers.count(kv.first)) fail("V5", "connection without a receiving thread block");
  for (auto& kv : receivers)
    if (!senders.count(kv.first)) fail("V5", "connection without a sending thread block");
  for (auto& kv : senders) {
    const ThreadBlock& st = a.gpus[kv.second.first].tbs[kv.second.second];
    const auto& rv = receivers[kv.first];
    const ThreadBlock& rt = a.gpus[rv.first].tbs[rv.second];
    std::vector<int> sc, rc;
    for (auto& in : st.steps)
      if (opRole(in.op).send) sc.push_back(in.cnt);
    for (auto& in : rt.steps)
      if (opRole(in.op).recv) rc.push_back(in.cnt);
    if (sc.size() != rc.size()) fail("V7", "connection: number of sends differs from number of receives");
    for (size_t k = 0; k < sc.size(); k++)
      if (sc[k] != rc[k]) fail("V7", "connection: k-th send and k-th receive carry different cnt");
  }
  // V11: the thread blocks holding multimem ops have the same ids on every rank (their
  // start / end group barrier pairs block b of every rank, reading R23)
  std::vector<int> mm0;
  for (auto& g : a.gpus) {
    std::vector<int> mm;
    for (auto& tb : g.tbs)
      for (auto& in : tb.steps)
        if (isMultimem(in.op)) {
          mm.push_back(tb.id);
          break;
        }
    if (!mm.empty() && a.proto != PROTO_SIMPLE) fail("V11", "multimem programs use the Simple protocol");
    if (g.id == 0) mm0 = mm;
    else if (mm != mm0) fail("V11", where(g.id, mm.empty() ? 0 : mm[0]) + ": multimem thread blocks differ from rank 0's");
  }
  deadlockCheck(a, slots, iters);
}

namespace {

// the instruction whose message receive step (tb, s) of rank g takes: the k-th send of the peer's
// thread block on this connection for the k-th receive of this one
const Instr* matchingSend(const Algo& a, int g, int tb, int s) {
  const ThreadBlock& rt = a.gpus[g].tbs[tb];
  if (rt.recv < 0) return nullptr;
  int k = 0;
  for (int i = 0; i < s; i++)
    if (opRole(rt.steps[i].op).recv) k++;
  for (auto& st : a.gpus[rt.recv].tbs) {
    if (st.send != g || st.chan != rt.chan) continue;
    int j = 0;
    for (auto& x : st.steps)
      if (opRole(x.op).send) {
        if (j == k) return &x;
        j++;
      }
  }
  return nullptr;
}

// Chunk k of a buffer has the length of chunk (k mod chunks-per-block) of every block (reading
// R1); scratch chunks are never short. A direct store of piece j of an instruction that also
// writes its own destination (rcs / rrcs) is cut to the receiver's chunk length, so that chunk
// must be as long as the sender's for every count: same position in its block, or scratch.
bool lengthsCompatible(const Algo& a, const Instr& snd, const Instr& rcv) {
  if (!opRole(snd.op).dst) return true;  // nothing local to shorten
  const int cb = a.gpus[0].iChunks / blocksOf(a.coll, BUF_IN, a.ngpus);
  if (cb <= 0) return false;
  for (int j = 0; j < rcv.cnt; j++) {
    if (rcv.dstBuf == BUF_SC) continue;
    if (snd.dstBuf == BUF_SC) return false;
    if ((snd.dstOff + j) % cb != (rcv.dstOff + j) % cb) return false;
  }
  return true;
}

// may receive step (tb, s) of rank g write its destination before its turn?
bool recvCanBeDirect(const Algo& a, int g, int tb, int s) {
  const GpuProgram& gp = a.gpus[g];
  const Instr& q = gp.tbs[tb].steps[s];
  if (q.op != OP_RECV && q.op != OP_RCS) return false;  // data must land unchanged
  const Instr* snd = matchingSend(a, g, tb, s);
  if (snd && !lengthsCompatible(a, *snd, q)) return false;
  auto canon = [&](int buf) { return (a.inplace && buf == BUF_OUT) ? BUF_IN : buf; };
  const int qb = canon(q.dstBuf);
  auto overlaps = [&](int buf, int off, int cnt) {
    return canon(buf) == qb && off < q.dstOff + q.cnt && q.dstOff < off + cnt;
  };
  for (auto& t : gp.tbs) {
    for (size_t k = 0; k < t.steps.size(); k++) {
      if (t.id == tb && (int)k == s) continue;
      const Instr& x = t.steps[k];
      OpRole ro = opRole(x.op);
      bool touches = (ro.src && overlaps(x.srcBuf, x.srcOff, x.cnt)) ||
                     ((ro.dst || x.op == OP_REDUCE) && overlaps(x.dstBuf, x.dstOff, x.cnt));
      if (!touches) continue;
      if (t.id == tb && (int)k > s) continue;  // same thread block, later in program order
      bool ordered = false;                     // waits on this receive (or a later step of its tb)
      for (auto& d : x.deps)
        if (d.first == tb && d.second >= s) ordered = true;
      if (!ordered) return false;
    }
  }
  return true;
}

// may receive step (tb, s) of rank g read its message straight from the sender's input chunk
// (reading R30)? The matching send is a plain `s` of an input chunk, the program is out of
// place and the sender's rank writes no input chunk, so the chunk holds the same data from the
// start of the launch to its end; Simple protocol only; a receive that is already direct keeps
// that. Every piece of the receive must have the length of the sender's chunk: its non-scratch
// chunks sit at the sender's chunk position in their block, and it has at least one.
bool recvCanPull(const Algo& a, int g, int tb, int s) {
  if (a.proto != PROTO_SIMPLE || a.inplace) return false;
  const ThreadBlock& rt = a.gpus[g].tbs[tb];
  const Instr& q = rt.steps[s];
  const Instr* snd = matchingSend(a, g, tb, s);
  if (!snd || snd->op != OP_SEND || snd->srcBuf != BUF_IN || snd->cnt != q.cnt) return false;
  if (recvCanBeDirect(a, g, tb, s)) return false;
  for (auto& t : a.gpus[rt.recv].tbs)
    for (auto& x : t.steps)
      if (opRole(x.op).dst && x.dstBuf == BUF_IN) return false;
  const int cb = a.gpus[0].iChunks / blocksOf(a.coll, BUF_IN, a.ngpus);
  if (cb <= 0) return false;
  const OpRole ro = opRole(q.op);
  for (int j = 0; j < q.cnt; j++) {
    const int want = (snd->srcOff + j) % cb;
    bool anchored = false;
    if (ro.src && q.srcBuf != BUF_SC) {
      if ((q.srcOff + j) % cb != want) return false;
      anchored = true;
    }
    if (ro.dst && q.dstBuf != BUF_SC) {
      if ((q.dstOff + j) % cb != want) return false;
      anchored = true;
    }
    if (!anchored) return false;
  }
  return true;
}

}  // namespace

DirectInfo directPlacement(const Algo& a, int rank) {
  DirectInfo di;
  const GpuProgram& g = a.gpus[rank];
  di.recvDirect.resize(g.tbs.size());
  di.sendDirect.resize(g.tbs.size());
  di.rdstBuf.resize(g.tbs.size());
  di.rdstOff.resize(g.tbs.size());
  di.rterminal.resize(g.tbs.size());
  di.recvPull.resize(g.tbs.size());
  di.pullOff.resize(g.tbs.size());
  di.sendPulled.resize(g.tbs.size());
  for (size_t t = 0; t < g.tbs.size(); t++) {
    const ThreadBlock& tb = g.tbs[t];
    di.recvDirect[t].assign(tb.steps.size(), 0);
    di.sendDirect[t].assign(tb.steps.size(), 0);
    di.rdstBuf[t].assign(tb.steps.size(), 0);
    di.rdstOff[t].assign(tb.steps.size(), 0);
    di.rterminal[t].assign(tb.steps.size(), 0);
    di.recvPull[t].assign(tb.steps.size(), 0);
    di.pullOff[t].assign(tb.steps.size(), 0);
    di.sendPulled[t].assign(tb.steps.size(), 0);
    for (size_t s = 0; s < tb.steps.size(); s++)
      if (opRole(tb.steps[s].op).recv) {
        di.recvDirect[t][s] = recvCanBeDirect(a, rank, (int)t, (int)s);
        if (recvCanPull(a, rank, (int)t, (int)s)) {
          di.recvPull[t][s] = 1;
          di.pullOff[t][s] = matchingSend(a, rank, (int)t, (int)s)->srcOff;
        }
      }
    if (tb.send < 0) continue;
    // pair the k-th send of (rank -> peer, chan) with the k-th receive of the peer's receiving tb
    const GpuProgram& pg = a.gpus[tb.send];
    const ThreadBlock* rt = nullptr;
    for (auto& x : pg.tbs)
      if (x.recv == rank && x.chan == tb.chan) rt = &x;
    if (!rt) continue;
    std::vector<int> rsteps;
    for (size_t k = 0; k < rt->steps.size(); k++)
      if (opRole(rt->steps[k].op).recv) rsteps.push_back((int)k);
    int k = 0;
    for (size_t s = 0; s < tb.steps.size(); s++) {
      if (!opRole(tb.steps[s].op).send) continue;
      if (k < (int)rsteps.size()) {
        int rs = rsteps[k];
        if (recvCanBeDirect(a, tb.send, rt->id, rs)) {
          di.sendDirect[t][s] = 1;
          di.rdstBuf[t][s] = rt->steps[rs].dstBuf;
          di.rdstOff[t][s] = rt->steps[rs].dstOff;
          di.rterminal[t][s] = rt->steps[rs].op == OP_RECV ? 1 : 0;
        }
        if (recvCanPull(a, tb.send, rt->id, rs)) di.sendPulled[t][s] = 1;
      }
      k++;
    }
  }
  return di;
}

}  // namespace msccl
