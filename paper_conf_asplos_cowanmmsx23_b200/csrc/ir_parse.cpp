// MSCCL-IR text parser (attribute-only XML subset, reading R0).
// Grammar: <algo ...> { <gpu ...> { <tb ...> { <step .../> } </tb> } </gpu> } </algo>
#include <cctype>
#include <cstdlib>
#include <map>

#include "ir.h"

namespace msccl {

namespace {

struct Tag {
  std::string name;
  bool closing = false;    // </name>
  bool selfClose = false;  // <name .../>
  std::map<std::string, std::string> attrs;
};

class Lexer {
 public:
  Lexer(const char* s, size_t n) : s_(s), n_(n) {}

  // Next tag; returns false at end of input. Skips text, comments and <?...?>.
  bool next(Tag& t) {
    for (;;) {
      while (i_ < n_ && s_[i_] != '<') {
        if (!isspace((unsigned char)s_[i_]) && s_[i_] != '\0') fail("unexpected text outside tags");
        i_++;
      }
      if (i_ >= n_) return false;
      if (startsWith("<!--")) {
        size_t e = find("-->", i_ + 4);
        i_ = e + 3;
        continue;
      }
      if (startsWith("<?")) {
        size_t e = find("?>", i_ + 2);
        i_ = e + 2;
        continue;
      }
      break;
    }
    t = Tag();
    i_++;  // '<'
    if (i_ < n_ && s_[i_] == '/') {
      t.closing = true;
      i_++;
    }
    t.name = ident();
    for (;;) {
      skipWs();
      if (i_ >= n_) fail("unterminated tag <" + t.name + ">");
      char c = s_[i_];
      if (c == '>') {
        i_++;
        return true;
      }
      if (c == '/' && i_ + 1 < n_ && s_[i_ + 1] == '>') {
        t.selfClose = true;
        i_ += 2;
        return true;
      }
      std::string k = ident();
      skipWs();
      if (i_ >= n_ || s_[i_] != '=') fail("expected '=' after attribute " + k);
      i_++;
      skipWs();
      if (i_ >= n_ || (s_[i_] != '"' && s_[i_] != '\'')) fail("expected quoted value for " + k);
      char q = s_[i_++];
      size_t st = i_;
      while (i_ < n_ && s_[i_] != q) i_++;
      if (i_ >= n_) fail("unterminated attribute value");
      t.attrs[k] = std::string(s_ + st, i_ - st);
      i_++;
    }
  }

 private:
  [[noreturn]] void fail(const std::string& m) { throw IRError("V1: " + m); }
  bool startsWith(const char* p) {
    size_t k = 0;
    while (p[k]) {
      if (i_ + k >= n_ || s_[i_ + k] != p[k]) return false;
      k++;
    }
    return true;
  }
  size_t find(const char* p, size_t from) {
    std::string hay(s_ + from, n_ - from);
    size_t r = hay.find(p);
    if (r == std::string::npos) fail("unterminated comment/declaration");
    return from + r;
  }
  void skipWs() {
    while (i_ < n_ && isspace((unsigned char)s_[i_])) i_++;
  }
  std::string ident() {
    size_t st = i_;
    while (i_ < n_ && (isalnum((unsigned char)s_[i_]) || s_[i_] == '_' || s_[i_] == '-')) i_++;
    if (st == i_) fail("expected a name");
    return std::string(s_ + st, i_ - st);
  }
  const char* s_;
  size_t n_, i_ = 0;
};

int toInt(const Tag& t, const char* key, bool required = true, int dflt = 0) {
  auto it = t.attrs.find(key);
  if (it == t.attrs.end()) {
    if (required) throw IRError(std::string("V1: <") + t.name + "> missing attribute '" + key + "'");
    return dflt;
  }
  const char* s = it->second.c_str();
  char* end = nullptr;
  long v = strtol(s, &end, 10);
  if (end == s || *end != '\0') throw IRError(std::string("V1: attribute ") + key + "='" + it->second + "' is not an integer");
  return (int)v;
}

std::vector<int> toList(const Tag& t, const char* key) {
  std::vector<int> out;
  auto it = t.attrs.find(key);
  if (it == t.attrs.end()) return out;
  const std::string& s = it->second;
  size_t i = 0;
  while (i < s.size()) {
    size_t j = s.find(',', i);
    if (j == std::string::npos) j = s.size();
    std::string tok = s.substr(i, j - i);
    if (!tok.empty()) {
      char* end = nullptr;
      long v = strtol(tok.c_str(), &end, 10);
      if (*end != '\0') throw IRError(std::string("V1: bad integer list ") + key);
      out.push_back((int)v);
    }
    i = j + 1;
  }
  return out;
}

int bufOf(const std::string& s) {
  if (s == "i") return BUF_IN;
  if (s == "o") return BUF_OUT;
  if (s == "s") return BUF_SC;
  if (s == "-" || s.empty()) return BUF_NONE;
  throw IRError("V1: unknown buffer '" + s + "'");
}

int opOf(const std::string& s) {
  static const char* names[OP_COUNT] = {"nop", "s", "r", "cpy", "re", "rrc", "rrs", "rrcs", "rcs", "mrd", "mst", "mrs"};
  for (int i = 0; i < OP_COUNT; i++)
    if (s == names[i]) return i;
  throw IRError("V1: unknown instruction type '" + s + "'");
}

std::string attr(const Tag& t, const char* k, const char* d = "") {
  auto it = t.attrs.find(k);
  return it == t.attrs.end() ? std::string(d) : it->second;
}

}  // namespace

Algo parseIR(const char* text, size_t len) {
  Lexer lx(text, len);
  Tag t;
  Algo a;
  if (!lx.next(t) || t.name != "algo" || t.closing) throw IRError("V1: root element must be <algo>");
  std::string coll = attr(t, "coll");
  if (coll == "allreduce") a.coll = COLL_ALLREDUCE;
  else if (coll == "allgather") a.coll = COLL_ALLGATHER;
  else if (coll == "reducescatter") a.coll = COLL_REDUCESCATTER;
  else if (coll == "alltoall") a.coll = COLL_ALLTOALL;
  else if (coll == "custom") a.coll = COLL_CUSTOM;
  else throw IRError("V1: unknown collective '" + coll + "'");
  std::string proto = attr(t, "proto", "Simple");
  if (proto == "Simple") a.proto = PROTO_SIMPLE;
  else if (proto == "LL") a.proto = PROTO_LL;
  else if (proto == "LL128") a.proto = PROTO_LL128;
  else throw IRError("V1: unknown protocol '" + proto + "'");
  a.name = attr(t, "name");
  a.ngpus = toInt(t, "ngpus");
  a.inplace = toInt(t, "inplace") != 0;
  a.aliassafe = toInt(t, "aliassafe", false, 0) != 0;
  a.nchannels = toInt(t, "nchannels", false, 1);
  if (t.selfClose) return a;
  GpuProgram* g = nullptr;
  ThreadBlock* tb = nullptr;
  while (lx.next(t)) {
    if (t.name == "algo" && t.closing) return a;
    if (t.name == "gpu") {
      if (t.closing) {
        g = nullptr;
        continue;
      }
      if (g) throw IRError("V1: nested <gpu>");
      a.gpus.emplace_back();
      g = &a.gpus.back();
      g->id = toInt(t, "id");
      g->iChunks = toInt(t, "i_chunks");
      g->oChunks = toInt(t, "o_chunks");
      g->sChunks = toInt(t, "s_chunks", false, 0);
      if (t.selfClose) g = nullptr;
    } else if (t.name == "tb") {
      if (t.closing) {
        tb = nullptr;
        continue;
      }
      if (!g || tb) throw IRError("V1: <tb> outside <gpu>");
      g->tbs.emplace_back();
      tb = &g->tbs.back();
      tb->id = toInt(t, "id");
      tb->send = toInt(t, "send");
      tb->recv = toInt(t, "recv");
      tb->chan = toInt(t, "chan");
      if (t.selfClose) tb = nullptr;
    } else if (t.name == "step") {
      if (!tb || t.closing) throw IRError("V1: <step> outside <tb>");
      Instr in;
      int s = toInt(t, "s");
      if (s != (int)tb->steps.size()) throw IRError("V1: steps must be numbered 0..n-1 in order");
      in.op = opOf(attr(t, "type"));
      in.srcBuf = bufOf(attr(t, "srcbuf", "-"));
      in.srcOff = toInt(t, "srcoff", false, -1);
      in.dstBuf = bufOf(attr(t, "dstbuf", "-"));
      in.dstOff = toInt(t, "dstoff", false, -1);
      in.cnt = toInt(t, "cnt", false, 1);
      std::vector<int> ids = toList(t, "depid"), ss = toList(t, "deps");
      if (ids.size() != ss.size()) throw IRError("V1: depid/deps length mismatch");
      for (size_t k = 0; k < ids.size(); k++)
        if (ids[k] >= 0) in.deps.push_back({ids[k], ss[k]});
      in.hasDep = toInt(t, "hasdep", false, 0) != 0;
      tb->steps.push_back(in);
    } else {
      throw IRError("V1: unexpected <" + t.name + ">");
    }
  }
  throw IRError("V1: missing </algo>");
}

int Algo::maxCnt() const {
  int m = 1;
  for (auto& g : gpus)
    for (auto& tb : g.tbs)
      for (auto& s : tb.steps) m = s.cnt > m ? s.cnt : m;
  return m;
}

bool Algo::hasReduce() const {
  for (auto& g : gpus)
    for (auto& tb : g.tbs)
      for (auto& s : tb.steps)
        if (s.op == OP_REDUCE || s.op == OP_RRC || s.op == OP_RRS || s.op == OP_RRCS || s.op == OP_MRD ||
            s.op == OP_MRS)
          return true;
  return false;
}

bool Algo::hasMultimem() const {
  for (auto& g : gpus)
    for (auto& tb : g.tbs)
      for (auto& s : tb.steps)
        if (isMultimem(s.op)) return true;
  return false;
}

}  // namespace msccl
