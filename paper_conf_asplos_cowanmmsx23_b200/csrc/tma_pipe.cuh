// TMA bulk-copy data path for one Simple-protocol message (sm_100a).
//
// A message (tile t of an instruction: `cnt` pieces) is streamed through a shared-memory
// ring of NST stages of CB bytes. Warp 0 is the mover: lane 0 issues 1-D bulk copies
// (cp.async.bulk, the TMA engine) global -> smem for the inputs (FIFO slot or dst = A,
// src = B) and smem -> global for the outputs (dst and/or the peer's FIFO slot); up to
// NST-1 stages of loads stay in flight per CTA without using registers. For instructions
// that reduce, the other warps combine A (+) B in shared memory between the load and the
// store. Stage reuse is ordered by cp.async.bulk.wait_group.read; load completion by
// per-stage mbarriers (complete_tx); reduction completion by per-stage mbarriers
// arrived by one lane of each compute warp. The interpreter semantics are unchanged:
// same elements, same single rounding per reduce (reading R6), same message boundaries.
// Included by interp.cuh inside namespace msccl (uses its vop/discardL2/policy helpers).
#pragma once

#ifndef MSCCL_TMA_CB
#define MSCCL_TMA_CB 16384  // bytes per stage and stream
#endif
#ifndef MSCCL_TMA_NST
#define MSCCL_TMA_NST 6     // stages
#endif
constexpr int TMA_CB = MSCCL_TMA_CB;
constexpr int TMA_NST = MSCCL_TMA_NST;
constexpr int TMA_SMEM = 2 * TMA_NST * TMA_CB + 2 * TMA_NST * 8 + 16;

__device__ __forceinline__ uint32_t smemAddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbarInit(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smemAddr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbarExpectTx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smemAddr(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbarArrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smemAddr(bar)) : "memory");
}
// Waits for the completion of the mbarrier phase with the given parity. These waits depend
// only on this CTA's own bulk copies and warps, so they cannot be blocked by a peer; a
// wait that exceeds 20 s is a kernel bug and traps instead of hanging the GPU.
__device__ __forceinline__ void mbarWait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  uint64_t t0 = 0;
  for (uint32_t it = 0; !done; it++) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smemAddr(bar)), "r"(parity)
        : "memory");
    if (!done && (it & 4095u) == 4095u) {
      uint64_t now = globaltimer();
      if (t0 == 0) t0 = now;
      else if (now - t0 > 20000000000ull) __trap();
    }
  }
}
__device__ __forceinline__ void tmaLoad(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smemAddr(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smemAddr(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void tmaStore(void* gdst, const void* ssrc, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(gdst),
               "r"(smemAddr(ssrc)), "r"(bytes), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void tmaCommit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void tmaWaitRead() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void tmaWaitAll() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fenceProxyAsyncShared() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fenceProxyAsyncGlobal() { asm volatile("fence.proxy.async.global;" ::: "memory"); }

struct TmaState {
  uint8_t* A;          // NST x CB
  uint8_t* B;          // NST x CB
  uint64_t* full;      // NST mbarriers: loads of a stage landed
  uint64_t* comp;      // NST mbarriers: reduction of a stage done
  uint32_t gc;         // chunks streamed so far by this CTA (phase bookkeeping)
};

// One piece: `bytes` (multiple of 16) of input(s) and output(s).
struct TmaPiece {
  const char* inA;  // FIFO slot or dst (reduce) — may be null for ops reading only src
  const char* inB;  // src for reductions; for pure copies the single input is inA
  char* out0;       // dst or nullptr
  char* out1;       // outgoing FIFO slot or nullptr
  int64_t bytes;
};

// Enumerate chunk q of the message: returns false past the end.
template <int MAXP>
__device__ __forceinline__ bool chunkOf(const TmaPiece* ps, int np, int q, int& pi, int64_t& off, uint32_t& sz) {
  for (int j = 0; j < np; j++) {
    int64_t nc = (ps[j].bytes + TMA_CB - 1) / TMA_CB;
    if (q < nc) {
      pi = j;
      off = (int64_t)q * TMA_CB;
      int64_t rem = ps[j].bytes - off;
      sz = (uint32_t)(rem < TMA_CB ? rem : TMA_CB);
      return true;
    }
    q -= (int)nc;
  }
  return false;
}

template <int MAXP>
__device__ __forceinline__ int totalChunks(const TmaPiece* ps, int np) {
  int n = 0;
  for (int j = 0; j < np; j++) n += (int)((ps[j].bytes + TMA_CB - 1) / TMA_CB);
  return n;
}

// Stream all pieces of a message. RED: the stage holds A and B and the compute warps
// write A = A (+) B before the store. DISCARD: inA is a FIFO slot whose consumed lines are
// dropped from L2. Called by every thread of the CTA; returns after all bulk stores of the
// message are complete (lane 0 of warp 0 waited for them).
template <int DT, int OP, bool RED, int MAXP>
__device__ __forceinline__ void tmaMessage(TmaState& s, const TmaPiece* ps, int np, bool discardA, int tid, int nt) {
  const int warp = tid >> 5, lane = tid & 31;
  const int N = totalChunks<MAXP>(ps, np);
  const uint32_t gc0 = s.gc;
  if (warp == 0) {
    uint64_t pFirst = 0, pLast = 0;
    if (lane == 0) {
      pFirst = policyEvictFirst();
      pLast = policyEvictLast();
      fenceProxyAsyncGlobal();  // generic acquire of the head counter -> async-proxy reads
    }
    auto issueLoad = [&](int q) {
      int pi;
      int64_t off;
      uint32_t sz;
      chunkOf<MAXP>(ps, np, q, pi, off, sz);
      const uint32_t st = (gc0 + (uint32_t)q) % TMA_NST;
      mbarExpectTx(&s.full[st], RED ? 2 * sz : sz);
      tmaLoad(s.A + (size_t)st * TMA_CB, ps[pi].inA + off, sz, &s.full[st], pFirst);
      if (RED) tmaLoad(s.B + (size_t)st * TMA_CB, ps[pi].inB + off, sz, &s.full[st], pFirst);
    };
    if (lane == 0)
      for (int q = 0; q < N && q < TMA_NST; q++) issueLoad(q);
    for (int q = 0; q < N; q++) {
      const uint32_t g = gc0 + (uint32_t)q;
      const uint32_t st = g % TMA_NST, par = (g / TMA_NST) & 1u;
      int pi;
      int64_t off;
      uint32_t sz;
      chunkOf<MAXP>(ps, np, q, pi, off, sz);
      mbarWait(&s.comp[st], par);  // compute warps arrive for every chunk (RED or not)
      if (lane == 0) {
        if (ps[pi].out0) tmaStore(ps[pi].out0 + off, s.A + (size_t)st * TMA_CB, sz, pFirst);
        if (ps[pi].out1) tmaStore(ps[pi].out1 + off, s.A + (size_t)st * TMA_CB, sz, pLast);
        tmaCommit();
      }
      if (discardA) {  // the slot lines are in smem now: drop them from L2 (no write-back)
        const char* base = ps[pi].inA + off;
        if ((((uintptr_t)base) & 127) == 0)
          for (uint32_t b = (uint32_t)lane * 128; b + 128 <= sz; b += 32 * 128) discardL2(base + b);
      }
      if (lane == 0 && q >= 1 && q - 1 + TMA_NST < N) {
        tmaWaitRead<1>();  // the stage of chunk q-1 has been read by its store
        issueLoad(q - 1 + TMA_NST);
      }
      __syncwarp();
    }
    if (lane == 0) {
      tmaWaitAll();
      fenceProxyAsyncGlobal();
    }
    __syncwarp();
  } else {
    // compute warps: combine A (+) B for reductions; for plain moves just pass the stage on,
    // so both mbarriers of a stage advance one phase per chunk whatever the instruction.
    const int ct = tid - 32, cn = nt - 32;
    for (int q = 0; q < N; q++) {
      const uint32_t g = gc0 + (uint32_t)q;
      const uint32_t st = g % TMA_NST, par = (g / TMA_NST) & 1u;
      int pi;
      int64_t off;
      uint32_t sz;
      chunkOf<MAXP>(ps, np, q, pi, off, sz);
      mbarWait(&s.full[st], par);
      uint4* a = reinterpret_cast<uint4*>(s.A + (size_t)st * TMA_CB);
      const uint4* b = reinterpret_cast<const uint4*>(s.B + (size_t)st * TMA_CB);
      if (RED) {
        for (uint32_t i = (uint32_t)ct; i < sz / 16; i += (uint32_t)cn) a[i] = vop<DT, OP>(a[i], b[i]);
        fenceProxyAsyncShared();  // generic smem writes -> async-proxy (bulk store) reads
      }
      __syncwarp();
      if (lane == 0) mbarArrive(&s.comp[st]);
    }
  }
  s.gc = gc0 + (uint32_t)N;
}

