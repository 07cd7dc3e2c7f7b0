// The MSCCL-IR interpreter kernel for sm_100a (MSCCLang §6.2, Fig. 5).
//
// One CTA = one IR thread block; every CTA of every rank on this GPU is co-resident
// (cooperative launch). Per CTA:
//
//   for t in [0, I):                      pipelining loop (Fig. 5 line 10)
//     for s in [0, nSteps):               instruction loop (line 12)
//       wait cross-TB deps                (lines 14-16; monotone semaphores, reading R4)
//       switch (op): primitive            (lines 18-23; one switch case per opcode)
//       post semaphore if hasDep          (lines 24-27)
//
// Primitives move tile t of each of the `cnt` chunks of the instruction (strided tiling,
// reading R3). Connections are receiver-side FIFOs of `slots` slots (§6.1):
//  * Simple: the sender waits for a free slot (ack counter), all threads store 16-byte
//    vectors straight into the receiver's slot (peer memory over NVLink, or the same HBM
//    for virtual ranks), then one thread fences and bumps the receiver's head counter;
//    the receiver acquires head, reads the slot with L1-bypassing loads, and acks.
//  * LL: 16-byte lines {data32, flag, data32, flag}; flag = message sequence number; the
//    receiver polls lines, no fence and no head counter (latency protocol).
// Reductions apply one correctly rounded binary op per element (reading R6).
#pragma once
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <stddef.h>
#include <stdint.h>
#include <type_traits>

#include "device.h"

namespace msccl {

enum { R_SUM = 0, R_PROD = 1, R_MAX = 2, R_MIN = 3, R_COPY = 4 };
enum { DT_I8 = 0, DT_U8 = 1, DT_I32 = 2, DT_U32 = 3, DT_I64 = 4, DT_U64 = 5, DT_F16 = 6, DT_F32 = 7, DT_F64 = 8,
       DT_BF16 = 9 };
enum { K_NOP = 0, K_SEND = 1, K_RECV = 2, K_COPY = 3, K_REDUCE = 4, K_RRC = 5, K_RRS = 6, K_RRCS = 7, K_RCS = 8,
       K_MRD = 9, K_MST = 10, K_MRS = 11 };
enum { KB_IN = 0, KB_OUT = 1, KB_SC = 2 };

struct V32 {  // 32-byte vector (one 256-bit LDG/STG on sm_100)
  uint4 a, b;
};

// ------------------------------------------------------------------ element types
template <int DT> struct DType;
#define MSCCL_INT_DTYPE(ID, S, U)                                                          \
  template <> struct DType<ID> {                                                           \
    typedef S T;                                                                           \
    static __device__ __forceinline__ T op(int o, T a, T b) {                              \
      if (o == R_SUM) return (T)((U)a + (U)b);                                             \
      if (o == R_PROD) return (T)((U)a * (U)b);                                            \
      if (o == R_MAX) return a >= b ? a : b;                                               \
      return a <= b ? a : b;                                                               \
    }                                                                                      \
  };
MSCCL_INT_DTYPE(DT_I8, int8_t, uint8_t)
MSCCL_INT_DTYPE(DT_U8, uint8_t, uint8_t)
MSCCL_INT_DTYPE(DT_I32, int32_t, uint32_t)
MSCCL_INT_DTYPE(DT_U32, uint32_t, uint32_t)
MSCCL_INT_DTYPE(DT_I64, int64_t, uint64_t)
MSCCL_INT_DTYPE(DT_U64, uint64_t, uint64_t)
#undef MSCCL_INT_DTYPE

// IEEE types: max/min follow numpy.maximum/minimum ((a >= b or a is NaN) ? a : b).
template <typename F>
__device__ __forceinline__ F fop(int o, F a, F b) {
  if (o == R_SUM) return a + b;
  if (o == R_PROD) return a * b;
  if (o == R_MAX) return (a >= b || a != a) ? a : b;
  return (a <= b || a != a) ? a : b;
}
template <> struct DType<DT_F32> {
  typedef float T;
  static __device__ __forceinline__ T op(int o, T a, T b) { return fop<float>(o, a, b); }
};
template <> struct DType<DT_F64> {
  typedef double T;
  static __device__ __forceinline__ T op(int o, T a, T b) { return fop<double>(o, a, b); }
};
template <> struct DType<DT_F16> {  // storage: IEEE binary16 bits
  typedef uint16_t T;
  static __device__ __forceinline__ T op(int o, T a, T b) {
    float x = __half2float(__ushort_as_half(a)), y = __half2float(__ushort_as_half(b));
    if (o == R_MAX) return (x >= y || x != x) ? a : b;
    if (o == R_MIN) return (x <= y || x != x) ? a : b;
    return __half_as_ushort(__float2half_rn(fop<float>(o, x, y)));
  }
};
template <> struct DType<DT_BF16> {  // storage: bf16 bits (top half of an fp32)
  typedef uint16_t T;
  static __device__ __forceinline__ float widen(T a) { return __uint_as_float(((uint32_t)a) << 16); }
  static __device__ __forceinline__ T op(int o, T a, T b) {
    float x = widen(a), y = widen(b);
    if (o == R_MAX) return (x >= y || x != x) ? a : b;
    if (o == R_MIN) return (x <= y || x != x) ? a : b;
    return __bfloat16_as_ushort(__float2bfloat16_rn(fop<float>(o, x, y)));
  }
};

// 16-byte vector op; sum/prod of fp16/bf16 use the packed correctly-rounded instructions.
template <int DT, int OP>
__device__ __forceinline__ uint4 vop(uint4 a, uint4 b) {
  typedef typename DType<DT>::T T;
  if (DT == DT_BF16 && (OP == R_SUM || OP == R_PROD)) {
    uint32_t* x = reinterpret_cast<uint32_t*>(&a);
    const uint32_t* y = reinterpret_cast<const uint32_t*>(&b);
#pragma unroll
    for (int i = 0; i < 4; i++) {
      __nv_bfloat162 p = *reinterpret_cast<__nv_bfloat162*>(&x[i]);
      __nv_bfloat162 q = *reinterpret_cast<const __nv_bfloat162*>(&y[i]);
      __nv_bfloat162 r = OP == R_SUM ? __hadd2(p, q) : __hmul2(p, q);
      x[i] = *reinterpret_cast<uint32_t*>(&r);
    }
    return a;
  }
  if (DT == DT_F16 && (OP == R_SUM || OP == R_PROD)) {
    uint32_t* x = reinterpret_cast<uint32_t*>(&a);
    const uint32_t* y = reinterpret_cast<const uint32_t*>(&b);
#pragma unroll
    for (int i = 0; i < 4; i++) {
      __half2 p = *reinterpret_cast<__half2*>(&x[i]);
      __half2 q = *reinterpret_cast<const __half2*>(&y[i]);
      __half2 r = OP == R_SUM ? __hadd2(p, q) : __hmul2(p, q);
      x[i] = *reinterpret_cast<uint32_t*>(&r);
    }
    return a;
  }
  T* x = reinterpret_cast<T*>(&a);
  const T* y = reinterpret_cast<const T*>(&b);
#pragma unroll
  for (int i = 0; i < (int)(16 / sizeof(T)); i++) x[i] = DType<DT>::op(OP, x[i], y[i]);
  return a;
}

template <int DT, int OP>
__device__ __forceinline__ V32 vop(V32 a, V32 b) {
  return V32{vop<DT, OP>(a.a, b.a), vop<DT, OP>(a.b, b.b)};
}

// ------------------------------------------------------------------ memory primitives
__device__ __forceinline__ uint4 ldcg(const void* p) {
  uint4 v;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void stg(void* p, uint4 v) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
// L2 cache policies: user input/output streams are touched once (evict_first); FIFO
// slots are written by the sender and read soon after by the receiver (evict_last), then
// discarded from L2 by the receiver so the dead slot is never written back to HBM.
#ifndef MSCCL_NO_HINTS
#define MSCCL_NO_HINTS 0
#endif
__device__ __forceinline__ uint64_t policyEvictFirst() {
  uint64_t p;
#if MSCCL_NO_HINTS
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
#else
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
#endif
  return p;
}
__device__ __forceinline__ uint64_t policyEvictNormal() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// drop a line's L2 priority back to normal (a forwarded line that was stored evict_last and
// has now been read by its forwarder: it is final output, no longer worth protecting)
__device__ __forceinline__ void demoteL2(const void* p) {
  asm volatile("applypriority.global.L2::evict_normal [%0], 128;" ::"l"(p) : "memory");
}
__device__ __forceinline__ uint64_t policyEvictLast() {
  uint64_t p;
#if MSCCL_NO_HINTS
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
#else
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
#endif
  return p;
}
template <int VB> struct VecT;
template <> struct VecT<16> { typedef uint4 T; };
template <> struct VecT<32> { typedef V32 T; };

// stream loads (user buffers): L1 bypass, L2 evict-first
__device__ __forceinline__ void ldStream(uint4& v, const void* p, uint64_t pol) {
  asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol) : "memory");
}
__device__ __forceinline__ void ldStream(V32& v, const void* p, uint64_t pol) {
  asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
               : "=r"(v.a.x), "=r"(v.a.y), "=r"(v.a.z), "=r"(v.a.w), "=r"(v.b.x), "=r"(v.b.y), "=r"(v.b.z),
                 "=r"(v.b.w) : "l"(p), "l"(pol) : "memory");
}
// FIFO loads: L2 only (the slot is rewritten by a peer between uses; never trust L1)
__device__ __forceinline__ void ldFifo(uint4& v, const void* p) {
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
}
__device__ __forceinline__ void ldFifo(V32& v, const void* p) {
  asm volatile("ld.global.cg.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v.a.x), "=r"(v.a.y), "=r"(v.a.z), "=r"(v.a.w), "=r"(v.b.x), "=r"(v.b.y), "=r"(v.b.z),
                 "=r"(v.b.w) : "l"(p) : "memory");
}
__device__ __forceinline__ void stHint(void* p, const uint4& v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w), "l"(pol) : "memory");
}
__device__ __forceinline__ void stHint(void* p, const V32& v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8}, %9;" ::"l"(p), "r"(v.a.x),
               "r"(v.a.y), "r"(v.a.z), "r"(v.a.w), "r"(v.b.x), "r"(v.b.y), "r"(v.b.z), "r"(v.b.w), "l"(pol)
               : "memory");
}
#ifndef MSCCL_NO_DISCARD
#define MSCCL_NO_DISCARD 0
#endif
__device__ __forceinline__ void discardL2(const void* p) {
#if !MSCCL_NO_DISCARD
  asm volatile("discard.global.L2 [%0], 128;" ::"l"(p) : "memory");
#endif
}

__device__ __forceinline__ uint4 ldvol(const void* p) {
  uint4 v;
  asm volatile("ld.volatile.global.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void stvol(void* p, uint4 v) {
  asm volatile("st.volatile.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ uint64_t ldAcquireSys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ldAcquireGpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void stRelaxedSys(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void stRelaxedGpu(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void fenceSys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
__device__ __forceinline__ void fenceGpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
#ifndef MSCCL_WARP_FENCE
#define MSCCL_WARP_FENCE 0
#endif
#ifndef MSCCL_REL_STORE
#define MSCCL_REL_STORE 0
#endif
__device__ __forceinline__ void postRelease(uint64_t* p, uint64_t v, bool sys) {
  if (sys) asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// post a connection counter (one u64 word in its own 128-byte line)
__device__ __forceinline__ void postFlag(uint64_t* p, uint64_t v, bool sys) {
  if (sys) stRelaxedSys(p, v);
  else stRelaxedGpu(p, v);
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// ------------------------------------------------------------------ watchdog + waits
struct Ctx {
  const KernelArgs* a;
  const RankArgs* ra;
  int tid, nt;
  // credit cache of the send connection (LL / LL128): the ack word is known to be >= ackKnown
  // (the receiver has consumed that many messages), so a send whose slot was freed by then
  // needs no flag read; uniform over the block. sAck: the ack value seen by the waiting thread.
  mutable uint64_t ackKnown;
  uint64_t* sAck;
  // direct placement (reading R15): the send peer's in/out/scratch base pointers in this
  // address space (shared memory; null = not reachable in this launch), and whether this
  // launch's ready handshake has been done (cross-launch mode; uniform over the block)
  char** peerDst;
  mutable bool readyDone;
  uint64_t sendL;  // thread 32: this launch's ordinal on the send connection
  char* (*mmBuf)[2];  // multimem ops: every rank's in/out base in this address space (shared memory)
};

static __device__ __noinline__ void raiseAbort(const KernelArgs& a) {
  for (int r = 0; r < a.nLocal; r++) {
    atomicExch(a.rank[r].abortFlag, 1u);
    *(volatile uint32_t*)a.rank[r].hostAbort = 1u;
  }
}

// Spin until *p >= target (acquire); `seen` = the value that satisfied the wait. Returns
// false on watchdog timeout / abort.
__device__ __forceinline__ bool waitGE(const uint64_t* p, uint64_t target, bool sys, const Ctx& c, uint64_t& seen) {
  if ((seen = (sys ? ldAcquireSys(p) : ldAcquireGpu(p))) >= target) return true;
  uint64_t t0 = globaltimer();
  for (uint32_t it = 1;; it++) {
    if ((seen = (sys ? ldAcquireSys(p) : ldAcquireGpu(p))) >= target) return true;
    if ((it & 1023u) == 0) {
      if (*(volatile uint32_t*)c.ra->abortFlag) return false;
      if (c.a->timeoutNs && globaltimer() - t0 > c.a->timeoutNs) {
        raiseAbort(*c.a);
        return false;
      }
    }
  }
}

__device__ __forceinline__ bool waitGE(const uint64_t* p, uint64_t target, bool sys, const Ctx& c) {
  uint64_t seen;
  return waitGE(p, target, sys, c, seen);
}

// Cross-thread-block dependency (Fig. 5 lines 15-16): wait until thread block dtb of this
// rank has finished step dstep of tile t in this launch (reading R4). A semaphore holds
// (launch generation mod 2^24) << 40 | (steps done in this launch); it can only hold this
// launch's value or the previous launch's, so the wait asks for the same generation field and
// at least the step -- a plain >= on the whole word broke after 2^24 launches, when the
// generation field wrapped below the previous launch's.
__device__ __forceinline__ bool waitDep(const RankArgs& ra, uint64_t dep, uint64_t gen, int t, const Ctx& c) {
  const int dtb = (int)(dep >> 48), dstep = (int)((dep >> 32) & 0xffff);
  const uint64_t dn = (uint32_t)dep;  // steps of thread block dtb
  const uint64_t want = (uint64_t)t * dn + (uint64_t)dstep + 1, g = gen << 40;
  const uint64_t* p = &ra.sem[dtb];
  constexpr uint64_t kLow = (1ull << 40) - 1;
  uint64_t v = ldAcquireGpu(p);
  if ((v & ~kLow) == g && (v & kLow) >= want) return true;
  const uint64_t t0 = globaltimer();
  for (uint32_t it = 1;; it++) {
    v = ldAcquireGpu(p);
    if ((v & ~kLow) == g && (v & kLow) >= want) return true;
    if ((it & 1023u) == 0) {
      if (*(volatile uint32_t*)c.ra->abortFlag) return false;
      if (c.a->timeoutNs && globaltimer() - t0 > c.a->timeoutNs) {
        raiseAbort(*c.a);
        return false;
      }
    }
  }
}

// ------------------------------------------------------------------ chunk geometry (reading R1)
__device__ __forceinline__ void chunkSpan(const KernelArgs& a, int buf, int64_t k, int64_t& start, int64_t& len) {
  if (buf == KB_SC) {
    start = k * a.E;
    len = a.E;
    return;
  }
  // chunk indices and chunks-per-block fit in 32 bits: a 32-bit division (a few instructions)
  // instead of the 64-bit division subroutine (hundreds of cycles on the latency path)
  const uint32_t kk = (uint32_t)k, cb = (uint32_t)a.cb;
  const uint32_t bq = kk / cb;
  int64_t b = (int64_t)bq, j = (int64_t)(kk - bq * cb);
  start = b * a.n + j * a.E;
  int64_t rem = a.n - j * a.E;
  len = rem < 0 ? 0 : (rem < a.E ? rem : a.E);
}

// ------------------------------------------------------------------ Simple-protocol piece
// out = RECV&&SRC ? op(recv, src) : REDDST ? op(dst, src) : RECV ? recv : src
// written to dst (DST) and/or the outgoing slot (SEND).
#ifndef MSCCL_TRACE
#define MSCCL_TRACE 0
#endif
#ifndef MSCCL_POST_LAST_WARP
#define MSCCL_POST_LAST_WARP 1
#endif
#ifndef MSCCL_UNROLL
#define MSCCL_UNROLL 4   // vectors in flight per lane and input stream (two input streams)
#endif
#ifndef MSCCL_UNROLL1
#define MSCCL_UNROLL1 8  // ... when the op reads one stream (copies, sends, receives): same registers
#endif

// Main vector loop: VB-byte vectors, U independent vectors in flight per thread.
// Returns the number of VB-byte vectors processed.
// store hint of one piece: a direct send whose receiver does not forward the data stores it
// L2 evict_first (reading R15, DI_SEND_TERMINAL)
// HINT_SRC_DEMOTE: the src lines were stored evict_last by a direct sender (forwarded data):
// demote them once read. HINT_SEND_NORMAL: store the outgoing lines evict_normal.
// HINT_NO_DISCARD: the received lines are not a FIFO slot (a pulled input chunk, reading R30).
enum { HINT_SEND_FIRST = 1, HINT_SRC_DEMOTE = 2, HINT_SEND_NORMAL = 4, HINT_NO_DISCARD = 8 };

template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST, int VB>
__device__ __forceinline__ int64_t vecLoop(int64_t nvec, const char* rslot, const char* src, char* dst, char* sslot,
                                           int ti, int nt, int hint) {
  typedef typename VecT<VB>::T Vec;
  constexpr int U = ((int)RECV + (int)SRC + (int)REDDST) >= 2 ? MSCCL_UNROLL : MSCCL_UNROLL1;
  const uint64_t pFirst = policyEvictFirst(), pLast0 = policyEvictLast();
  const uint64_t pLast = (hint & HINT_SEND_FIRST) ? pFirst : (hint & HINT_SEND_NORMAL) ? policyEvictNormal() : pLast0;
  const bool canDiscard = RECV && !(hint & HINT_NO_DISCARD) && ((((uintptr_t)rslot) & 127) == 0);
  const int lane = ti & 31, warp = ti >> 5, nw = nt >> 5;
  // Full blocks of U x 32 vectors, one block per warp-iteration (warp-uniform trip count,
  // so the __syncwarp below is reached by every lane); each u-row is 32 x VB contiguous bytes.
  const int64_t nblk = nvec / (U * 32);
  for (int64_t blk = warp; blk < nblk; blk += nw) {
    const int64_t base = blk * (U * 32) + lane;
    Vec x[U], y[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      if constexpr (RECV) ldFifo(x[u], rslot + (base + u * 32) * VB);
      if constexpr (REDDST) ldStream(x[u], dst + (base + u * 32) * VB, pFirst);
      if constexpr (SRC) ldStream(y[u], src + (base + u * 32) * VB, pFirst);
    }
#pragma unroll
    for (int u = 0; u < U; u++) {
      Vec v;
      if constexpr ((RECV && SRC) || REDDST) v = vop<DT, OP>(x[u], y[u]);
      else if constexpr (RECV) v = x[u];
      else v = y[u];
      if constexpr (DST) stHint(dst + (base + u * 32) * VB, v, pFirst);
      if constexpr (SEND) stHint(sslot + (base + u * 32) * VB, v, pLast);
    }
    if constexpr (RECV) {
      // every lane's loads of this block have been consumed: drop the dead slot lines
      __syncwarp();
      if (canDiscard && ((lane * VB) & 127) == 0) {
#pragma unroll
        for (int u = 0; u < U; u++) discardL2(rslot + (base + u * 32) * VB);
      }
    }
    if constexpr (SRC && !RECV && !REDDST) {
      if ((hint & HINT_SRC_DEMOTE) && ((lane * VB) & 127) == 0) {
#pragma unroll
        for (int u = 0; u < U; u++) demoteL2(src + (base + u * 32) * VB);
      }
    }
  }
  for (int64_t i = nblk * (U * 32) + ti; i < nvec; i += nt) {
    Vec x, y, v;
    if constexpr (RECV) ldFifo(x, rslot + i * VB);
    if constexpr (REDDST) ldStream(x, dst + i * VB, pFirst);
    if constexpr (SRC) ldStream(y, src + i * VB, pFirst);
    if constexpr ((RECV && SRC) || REDDST) v = vop<DT, OP>(x, y);
    else if constexpr (RECV) v = x;
    else v = y;
    if constexpr (DST) stHint(dst + i * VB, v, pFirst);
    if constexpr (SEND) stHint(sslot + i * VB, v, pLast);
  }
  return nvec;
}

// ------------------------------------------------------------------ Simple-protocol piece
// out = RECV&&SRC ? op(recv, src) : REDDST ? op(dst, src) : RECV ? recv : src
// written to dst (DST) and/or the outgoing slot (SEND). Threads ti of [0, nt): the whole
// block (nt = blockDim) or one warp (nt = 32, warp flags).
template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST>
__device__ __forceinline__ void pieceSimple(int64_t m, const char* rslot, const char* src, char* dst, char* sslot,
                                            int ti, int nt, int hint = 0) {
  typedef typename DType<DT>::T T;
  const int64_t bytes = m * (int64_t)sizeof(T);
  uintptr_t al = (uintptr_t)rslot | (uintptr_t)src | (uintptr_t)dst | (uintptr_t)sslot;
  int64_t done = 0;  // bytes handled by the vector paths
  if ((al & 31) == 0) {
    done = 32 * vecLoop<DT, OP, RECV, SEND, SRC, DST, REDDST, 32>(bytes / 32, rslot, src, dst, sslot, ti, nt, hint);
  } else if ((al & 15) == 0) {
    done = 16 * vecLoop<DT, OP, RECV, SEND, SRC, DST, REDDST, 16>(bytes / 16, rslot, src, dst, sslot, ti, nt, hint);
  }
  if ((al & 15) == 0 && bytes - done >= 16) {  // 16-byte remainder after the 32-byte path
    const int64_t off = done;
    const int64_t nv = (bytes - done) / 16;
    done += 16 * vecLoop<DT, OP, RECV, SEND, SRC, DST, REDDST, 16>(
                     nv, RECV ? rslot + off : nullptr, SRC ? src + off : nullptr, (DST || REDDST) ? dst + off : nullptr,
                     SEND ? sslot + off : nullptr, ti, nt, hint);
  }
  // scalar tail (ragged chunk end or unaligned buffers)
  for (int64_t e = done / (int64_t)sizeof(T) + ti; e < m; e += nt) {
    T x = 0, y = 0, v;
    if constexpr (RECV) x = *(volatile const T*)(rslot + e * sizeof(T));
    if constexpr (REDDST) x = *(volatile const T*)(dst + e * sizeof(T));
    if constexpr (SRC) y = *(volatile const T*)(src + e * sizeof(T));
    if constexpr ((RECV && SRC) || REDDST) v = DType<DT>::op(OP, x, y);
    else if constexpr (RECV) v = x;
    else v = y;
    if constexpr (DST) *(volatile T*)(dst + e * sizeof(T)) = v;
    if constexpr (SEND) *(volatile T*)(sslot + e * sizeof(T)) = v;
  }
}

// ------------------------------------------------------------------ LL-protocol piece
// Payload travels in 8-byte units inside 16-byte lines {lo32, flag, hi32, flag}.
// user-buffer units for LL128 (not concurrently written by peers): plain cached accesses
__device__ __forceinline__ uint64_t loadUnitPlain(const char* p, int64_t bytes) {
  if (bytes == 8 && (((uintptr_t)p) & 7) == 0) return *(const uint64_t*)p;
  uint64_t v = 0;
  for (int64_t k = 0; k < bytes; k++) v |= (uint64_t)(*(const uint8_t*)(p + k)) << (8 * k);
  return v;
}
__device__ __forceinline__ void storeUnitPlain(char* p, uint64_t v, int64_t bytes) {
  if (bytes == 8 && (((uintptr_t)p) & 7) == 0) {
    *(uint64_t*)p = v;
    return;
  }
  for (int64_t k = 0; k < bytes; k++) *(uint8_t*)(p + k) = (uint8_t)(v >> (8 * k));
}
__device__ __forceinline__ uint64_t loadUnit(const char* p, int64_t bytes) {
  if (bytes == 8 && (((uintptr_t)p) & 7) == 0) return *(volatile const uint64_t*)p;
  uint64_t v = 0;
  for (int64_t k = 0; k < bytes; k++) v |= (uint64_t)(*(volatile const uint8_t*)(p + k)) << (8 * k);
  return v;
}
__device__ __forceinline__ void storeUnit(char* p, uint64_t v, int64_t bytes) {
  if (bytes == 8 && (((uintptr_t)p) & 7) == 0) {
    *(volatile uint64_t*)p = v;
    return;
  }
  for (int64_t k = 0; k < bytes; k++) *(volatile uint8_t*)(p + k) = (uint8_t)(v >> (8 * k));
}
template <int DT, int OP>
__device__ __forceinline__ uint64_t unitOp(uint64_t a, uint64_t b) {
  typedef typename DType<DT>::T T;
  T* x = reinterpret_cast<T*>(&a);
  const T* y = reinterpret_cast<const T*>(&b);
#pragma unroll
  for (int i = 0; i < (int)(8 / sizeof(T)); i++) x[i] = DType<DT>::op(OP, x[i], y[i]);
  return a;
}

// Every LL piece message has exactly `sendUnits` lines: ceil(min(T, E - t*T) * w / 8), the
// width of this tile of a FULL chunk, whatever the sender's own chunk length (reading R2:
// a ragged in/out chunk may be received into a full-length scratch chunk, whose receiver
// polls more lines than the sender has data for; the sender pads with zeros).
template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST>
__device__ __forceinline__ bool pieceLL(int64_t m, int64_t sendUnits, const char* rslot, const char* src, char* dst,
                                        char* sslot, uint32_t rflag, uint32_t sflag, const Ctx& c) {
  typedef typename DType<DT>::T T;
  const int64_t bytes = m > 0 ? m * (int64_t)sizeof(T) : 0;
  const int64_t units = (bytes + 7) / 8;
  const int64_t total = SEND ? (units > sendUnits ? units : sendUnits) : units;
  bool ok = true;
  for (int64_t u = c.tid; u < total; u += c.nt) {
    const bool has = u < units;
    const int64_t off = u * 8;
    const int64_t nb = has ? (bytes - off < 8 ? bytes - off : 8) : 0;
    uint64_t x = 0, y = 0, v = 0;
    // the local operand first: its load overlaps the wait for the incoming line
    if (has) {
      if constexpr (REDDST) x = loadUnit(dst + off, nb);
      if constexpr (SRC) y = loadUnit(src + off, nb);
    }
    if constexpr (RECV) {
      if (has) {
        const char* line = rslot + u * 16;
        uint4 l = ldvol(line);
        if (l.y != rflag || l.w != rflag) {
          uint64_t t0 = globaltimer();
          for (uint32_t it = 1;; it++) {
            l = ldvol(line);
            if (l.y == rflag && l.w == rflag) break;
            if ((it & 1023u) == 0) {
              if (*(volatile uint32_t*)c.ra->abortFlag) { ok = false; break; }
              if (c.a->timeoutNs && globaltimer() - t0 > c.a->timeoutNs) { raiseAbort(*c.a); ok = false; break; }
            }
          }
          if (!ok) break;
        }
        x = (uint64_t)l.x | ((uint64_t)l.z << 32);
      }
    }
    if (has) {
      if constexpr ((RECV && SRC) || REDDST) v = unitOp<DT, OP>(x, y);
      else if constexpr (RECV) v = x;
      else v = y;
      if constexpr (DST) storeUnit(dst + off, v, nb);
    }
    if constexpr (SEND) stvol(sslot + u * 16, make_uint4((uint32_t)v, sflag, (uint32_t)(v >> 32), sflag));
  }
  return ok;
}

// ------------------------------------------------------------------ LL128-protocol piece
// 128-byte lines written by 8 lanes x 16 bytes in one warp store: lanes 0-6 carry 16 payload
// bytes, lane 7 carries 8 payload bytes and the 64-bit flag (message sequence number), so a
// line holds 120 payload bytes (LL128 sits between LL and Simple). A line is
// read by the same 8 lanes in one warp load and accepted when its flag matches; no fence and
// no separate head counter are needed. Lines per piece message: ceil(min(T, E - t*T)*w/120)
// (the sender pads, reading R2).
#ifndef MSCCL_LL128_BACKOFF
#define MSCCL_LL128_BACKOFF 8  // empty polls of a batch before the poller sleeps between polls
#endif
#ifndef MSCCL_LL128_UNROLL
#define MSCCL_LL128_UNROLL 4  // lines in flight per 8-lane group of a warp
#endif
// One batch of 4*U lines of a warp (8 lanes per line, U lines per lane group). FULL: every
// line of the batch carries 120 payload bytes and the user pointers are 8-byte aligned, so
// the payload moves as plain 8-byte words (no ragged-edge logic).
template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool FULL>
__device__ __forceinline__ bool ll128Batch(int64_t base, int64_t bytes, int64_t lines, int64_t total, const char* rslot,
                                           const char* src, char* dst, char* sslot, uint64_t rflag, uint64_t sflag,
                                           int g, int sub, const Ctx& c) {
  constexpr int U = MSCCL_LL128_UNROLL;
  const int64_t lb = g == 7 ? 8 : 16;  // payload bytes of this lane in a line
  // 1. the local operand of every line this lane owns, loaded before the flag poll so its
  //    latency overlaps the wait for the incoming line
  uint64_t b0[U], b1[U];
#pragma unroll
  for (int u = 0; u < U; u++) {
    b0[u] = b1[u] = 0;
    if constexpr (SRC) {
      const int64_t po = (base + u * 4 + sub) * 120 + g * 16;
      if (FULL) {
        b0[u] = *(const uint64_t*)(src + po);
        if (g != 7) b1[u] = *(const uint64_t*)(src + po + 8);
      } else {
        int64_t nb = bytes - po;
        nb = nb < 0 ? 0 : (nb > lb ? lb : nb);
        if (nb > 0) {
          const int64_t nb0 = nb > 8 ? 8 : nb;
          b0[u] = loadUnitPlain(src + po, nb0);
          if (nb > 8) b1[u] = loadUnitPlain(src + po + 8, nb - 8);
        }
      }
    }
  }
  // 2. the incoming lines: poll until every line of the batch carries this message's flag
  uint64_t x0[U], x1[U];
  if constexpr (RECV) {
    uint4 l[U];
    uint64_t t0 = 0;
    for (uint32_t it = 0;; it++) {
      bool mine = true;
#pragma unroll
      for (int u = 0; u < U; u++) {
        const int64_t L = base + u * 4 + sub;
        if (FULL || L < lines) {
          l[u] = ldvol(rslot + L * 128 + g * 16);
          if (g == 7 && ((uint64_t)l[u].z | ((uint64_t)l[u].w << 32)) != rflag) mine = false;
        }
      }
      if (__all_sync(0xffffffffu, mine)) break;
      if (it >= MSCCL_LL128_BACKOFF) __nanosleep(64);  // back off after empty polls (L2 traffic)
      if ((it & 255u) == 255u) {
        uint64_t now = globaltimer();
        if (t0 == 0) t0 = now;
        if (*(volatile uint32_t*)c.ra->abortFlag) return false;
        if (c.a->timeoutNs && now - t0 > c.a->timeoutNs) {
          raiseAbort(*c.a);
          return false;
        }
      }
    }
#pragma unroll
    for (int u = 0; u < U; u++) {
      x0[u] = (uint64_t)l[u].x | ((uint64_t)l[u].y << 32);
      x1[u] = (uint64_t)l[u].z | ((uint64_t)l[u].w << 32);
    }
  }
  // 3. combine; store to dst and/or the outgoing lines
#pragma unroll
  for (int u = 0; u < U; u++) {
    const int64_t L = base + u * 4 + sub;
    if (!FULL && L >= total) continue;
    const int64_t po = L * 120 + g * 16;
    int64_t nb = lb;
    if (!FULL) {
      nb = bytes - po;
      nb = nb < 0 ? 0 : (nb > lb ? lb : nb);
    }
    uint64_t v0 = 0, v1 = 0;
    if constexpr (RECV && SRC) {  // op(received, local), as in every protocol
      v0 = unitOp<DT, OP>(x0[u], b0[u]);
      v1 = unitOp<DT, OP>(x1[u], b1[u]);
    } else if constexpr (RECV) {
      v0 = x0[u];
      v1 = x1[u];
    } else {
      v0 = b0[u];
      v1 = b1[u];
    }
    if constexpr (DST) {
      if (FULL) {
        *(uint64_t*)(dst + po) = v0;
        if (g != 7) *(uint64_t*)(dst + po + 8) = v1;
      } else if (nb > 0) {
        const int64_t nb0 = nb > 8 ? 8 : nb;
        storeUnitPlain(dst + po, v0, nb0);
        if (nb > 8) storeUnitPlain(dst + po + 8, v1, nb - 8);
      }
    }
    if constexpr (SEND) {
      if (nb == 0) v0 = 0;  // padding line (R2): deterministic zeros
      if (nb <= 8) v1 = 0;
      if (g == 7) v1 = sflag;
      stvol(sslot + L * 128 + g * 16, make_uint4((uint32_t)v0, (uint32_t)(v0 >> 32), (uint32_t)v1, (uint32_t)(v1 >> 32)));
    }
  }
  return true;
}

template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST>
__device__ __forceinline__ bool pieceLL128(int64_t m, int64_t sendLines, const char* rslot, const char* src, char* dst,
                                           char* sslot, uint64_t rflag, uint64_t sflag, const Ctx& c) {
  typedef typename DType<DT>::T T;
  static_assert(!REDDST, "local reduces take the Simple path");
  constexpr int U = MSCCL_LL128_UNROLL;
  const int64_t bytes = m > 0 ? m * (int64_t)sizeof(T) : 0;
  const int64_t lines = (bytes + 119) / 120;
  const int64_t total = SEND ? (lines > sendLines ? lines : sendLines) : lines;
  const int lane = c.tid & 31, warp = c.tid >> 5, nw = c.nt >> 5;
  const int g = lane & 7, sub = lane >> 3;
  const bool aligned = ((((uintptr_t)src) | ((uintptr_t)dst)) & 7) == 0;
  for (int64_t base = (int64_t)warp * 4 * U; base < total; base += (int64_t)nw * 4 * U) {
    bool ok;
    if (aligned && (base + 4 * U) * 120 <= bytes)
      ok = ll128Batch<DT, OP, RECV, SEND, SRC, DST, true>(base, bytes, lines, total, rslot, src, dst, sslot, rflag, sflag,
                                                          g, sub, c);
    else
      ok = ll128Batch<DT, OP, RECV, SEND, SRC, DST, false>(base, bytes, lines, total, rslot, src, dst, sslot, rflag,
                                                           sflag, g, sub, c);
    if (!ok) return false;
  }
  return true;
}

// ------------------------------------------------------------------ per-protocol piece loops
#define MSCCL_PIECE_GEOM                                                                  \
  const KernelArgs& a = *c.a;                                                             \
  const RankArgs& ra = *c.ra;                                                             \
  const int64_t w = sizeof(typename DType<DT>::T);                                        \
  const int64_t a0 = (int64_t)t * a.T;

// piece j of the instruction at tile t: element count m and src/dst pointers (reading R2)
template <int DT, bool SRC, bool DST, bool REDDST>
__device__ __forceinline__ int64_t pieceGeom(const Ctx& c, const DevInstr& in, int t, int j, const char*& src, char*& dst) {
  MSCCL_PIECE_GEOM
  int64_t ss = 0, sl = INT64_MAX, ds = 0, dl = INT64_MAX;
  if (SRC) chunkSpan(a, in.srcBuf, (int64_t)in.srcOff + j, ss, sl);
  if (DST || REDDST) chunkSpan(a, in.dstBuf, (int64_t)in.dstOff + j, ds, dl);
  int64_t L = sl < dl ? sl : dl;
  int64_t hi = a0 + a.T < L ? a0 + a.T : L;
  src = SRC ? ra.buf[in.srcBuf] + (ss + a0) * w : nullptr;
  dst = (DST || REDDST) ? ra.buf[in.dstBuf] + (ds + a0) * w : nullptr;
  return hi - a0;
}

// Cross-launch direct placement (a.direct == 2, reading R15b): before its first direct store of
// a launch, the sender's thread 32 waits until the receiving thread block of THIS launch has
// published its destination references on the connection's ready line (so the receiver's
// stream has finished every earlier use of that buffer), then resolves them into pointers of
// this process (raw pointer for single-process communicators, registered-buffer table entry
// for CUDA IPC peers). A zero reference means "not reachable": the connection falls back to
// the FIFO for this launch, and the receiver (which published the zero) does the same.
__device__ __forceinline__ char* resolveRef(const RankArgs& ra, int peer, uint64_t ref) {
  if (ref == 0) return nullptr;
  if (!(ref & MSCCL_REF_REG)) return (char*)ref;  // raw pointer (one address space)
  const uint32_t idx = (uint32_t)((ref >> 40) & 0x7fffffu);
  const uint64_t off = ref & ((1ull << 40) - 1);
  if (idx >= (uint32_t)ra.regMax) return nullptr;
  char* base = ra.regMap[(size_t)peer * ra.regMax + idx];
  return base ? base + off : nullptr;
}

__device__ __forceinline__ bool waitReady(const Ctx& c, const DevTB& tb) {
  uint64_t seen;
  if (!waitGE(tb.sendReady, c.sendL, c.a->sysScope != 0, c, seen)) return false;
  if (*(volatile const uint64_t*)(tb.sendReady + 4) != (uint64_t)c.a->T) {  // ranks chose different tiles
    raiseAbort(*c.a);                                                        // (asymmetric registration, R19)
    return false;
  }
  bool any = false;
#pragma unroll
  for (int b = 0; b < 3; b++) {
    const uint64_t ref = *(volatile const uint64_t*)(tb.sendReady + 1 + b);
    c.peerDst[b] = resolveRef(*c.ra, tb.sendPeer, ref);
    if (ref && !c.peerDst[b]) {  // published but not mapped here: the receiver expects a direct store
      raiseAbort(*c.a);          // that this sender cannot make (registration not connected)
      return false;
    }
    any = any || c.peerDst[b] != nullptr;
  }
  if (any) atomicAdd(c.ra->stats, 1ull);
  return true;
}

// is this send / receive a direct placement in this launch (reading R15)?
__device__ __forceinline__ bool sendIsDirect(const Ctx& c, const DevInstr& in) {
  return (in.flags & DI_SEND_DIRECT) && c.a->direct && (c.a->direct == 1 || c.peerDst[in.rdstBuf] != nullptr);
}
__device__ __forceinline__ bool recvIsDirect(const Ctx& c, const DevInstr& in) {
  return (in.flags & DI_RECV_DIRECT) && c.a->direct && ((c.ra->directMask >> in.dstBuf) & 1);
}
// reading R30: every rank in this launch and MSCCL_DIRECT_HINTS bit 4 (both ends see the same
// launch arguments, so they agree)
__device__ __forceinline__ bool pullOn(const Ctx& c) { return c.a->direct == 1 && (c.a->directHints & 16); }

template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST>
__device__ __noinline__ void movePiecesSimple(const Ctx& c, const DevTB& tb, const DevInstr& in, int t,
                                              const char* rslot, char* sslot) {
  MSCCL_PIECE_GEOM
  if (SEND && !RECV && (in.flags & DI_SEND_PULLED) && pullOn(c)) return;  // the receiver reads the chunk
  const bool sdirect = SEND && sendIsDirect(c, in);
  const bool rdirect = RECV && recvIsDirect(c, in);
  const bool rpull = RECV && (in.flags & DI_RECV_PULL) && pullOn(c);
  for (int j = 0; j < in.cnt; j++) {
    const char* src;
    char* dst;
    int64_t m = pieceGeom<DT, SRC, DST, REDDST>(c, in, t, j, src, dst);
    char* so = SEND ? sslot + j * a.T * w : nullptr;
    const char* ri = RECV ? rslot + j * a.T * w : nullptr;
    if (rpull) {  // reading R30: the message is the sender's input chunk, unchanged for the launch
      int64_t ps, pl;
      chunkSpan(a, 0, (int64_t)in.pullOff + j, ps, pl);  // buffer 0 = in
      ri = a.rank[in.chainLen].buf[0] + (ps + a0) * w;
      if (pl - a0 < m) m = pl - a0;
    }
    if (sdirect) {  // reading R15: write straight into the receiver's destination chunk
      int64_t rs, rl;
      chunkSpan(a, in.rdstBuf, (int64_t)in.rdstOff + j, rs, rl);
      so = c.peerDst[in.rdstBuf] + (rs + a0) * w;
      if (rl - a0 < m) m = rl - a0;
    }
    if (m <= 0) continue;
    int hint = (sdirect && (in.flags & DI_SEND_TERMINAL)) ? (a.directHints & HINT_SEND_FIRST) : 0;
    if (SEND && !(hint & HINT_SEND_FIRST)) {  // MSCCL_DIRECT_HINTS bit 2: FIFO stores, bit 3: direct forwards
      if (sdirect ? (a.directHints & 8) : (a.directHints & 4)) hint |= HINT_SEND_NORMAL;
    }
    if (rdirect) {  // the data is already in dst (the sender wrote it there)
      if (SEND)
        pieceSimple<DT, OP, false, true, true, false, false>(m, nullptr, dst, nullptr, so, c.tid, c.nt,
                                                             hint | (a.directHints & HINT_SRC_DEMOTE));
      continue;
    }
    pieceSimple<DT, OP, RECV, SEND, SRC, DST, REDDST>(m, ri, src, dst, so, c.tid, c.nt,
                                                      rpull ? hint | HINT_NO_DISCARD : hint);
  }
}

template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST>
__device__ __noinline__ bool movePiecesLL(const Ctx& c, const DevInstr& in, int t, const char* rslot, char* sslot,
                                          uint64_t rseq, uint64_t sseq) {
  MSCCL_PIECE_GEOM
  bool ok = true;
  for (int j = 0; j < in.cnt; j++) {
    const char* src;
    char* dst;
    const int64_t m = pieceGeom<DT, SRC, DST, REDDST>(c, in, t, j, src, dst);
    const int64_t lineOff = j * ((a.T * w + 7) / 8) * 16;
    const int64_t full = a.E - a0 < a.T ? a.E - a0 : a.T;
    ok &= pieceLL<DT, OP, RECV, SEND, SRC, DST, REDDST>(m, (full * w + 7) / 8, RECV ? rslot + lineOff : nullptr, src, dst,
                                                      SEND ? sslot + lineOff : nullptr, (uint32_t)rseq, (uint32_t)sseq, c);
  }
  return ok;
}

template <int DT, int OP, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST>
__device__ __noinline__ bool movePiecesLL128(const Ctx& c, const DevInstr& in, int t, const char* rslot, char* sslot,
                                             uint64_t rseq, uint64_t sseq) {
  MSCCL_PIECE_GEOM
  bool ok = true;
  const int64_t linesPer = (a.T * w + 119) / 120;
  const int64_t full = a.E - a0 < a.T ? a.E - a0 : a.T;
  for (int j = 0; j < in.cnt; j++) {
    const char* src;
    char* dst;
    const int64_t m = pieceGeom<DT, SRC, DST, REDDST>(c, in, t, j, src, dst);
    ok &= pieceLL128<DT, OP, RECV, SEND, SRC, DST, REDDST>(m, (full * w + 119) / 120,
                                                         RECV ? rslot + j * linesPer * 128 : nullptr, src, dst,
                                                         SEND ? sslot + j * linesPer * 128 : nullptr, rseq, sseq, c);
  }
  return ok;
}

// FIFO slot of message number x (monotone 64-bit counter): a mask for power-of-two slot counts
// (the default 4), the 64-bit remainder otherwise
__device__ __forceinline__ uint32_t slotOf(uint64_t x, uint32_t s) {
  return (s & (s - 1)) == 0 ? (uint32_t)x & (s - 1) : (uint32_t)(x % s);
}

// ------------------------------------------------------------------ one instruction, one tile
template <int DT, int OP, int PROTO, bool RECV, bool SEND, bool SRC, bool DST, bool REDDST>
__device__ __noinline__ bool runOp(const Ctx& c, const DevTB& tb, const DevInstr& in, int t, uint64_t& sent,
                                   uint64_t& recvd, volatile int* sAbort) {
  const KernelArgs& a = *c.a;
  constexpr bool ll = PROTO != 0;  // LL / LL128: the flags travel inside the data lines
  bool ok = true;
  const bool sys = a.sysScope != 0;  // virtual ranks on one GPU only need gpu-scope ordering
#if MSCCL_TRACE
  uint64_t tr0 = c.tid == 0 ? globaltimer() : 0, tr1 = 0, tr2 = 0, tr3 = 0, tr4 = 0;
#endif
  if (RECV && !ll && c.tid == 0) ok = waitGE(tb.recvHead, recvd + 1, sys, c);
#if MSCCL_TRACE
  if (c.tid == 0) tr1 = globaltimer();
#endif
  // a free slot: at most `slots` messages posted and not yet consumed (§6.1)
  // (a direct message uses no slot: no credit needed, reading R15)
  // LL / LL128: credits already seen (c.ackKnown) are not re-read, so a step that has its slot
  // (no head to wait for: the flags travel in the lines) starts moving data without a flag
  // round trip or barrier. Simple keeps the per-message check (it needs the barrier anyway).
  if constexpr (!ll) {
    if (SEND && a.direct == 2 && (in.flags & DI_SEND_DIRECT) && !c.readyDone) {
      if (c.tid == 32) ok = waitReady(c, tb);  // first direct store of this launch on this connection
      __syncthreads();                         // c.peerDst visible to every thread
      c.readyDone = true;
    }
    if (SEND && c.tid == 32 && sent + 1 > (uint64_t)a.slots && !sendIsDirect(c, in) &&
        !((in.flags & DI_SEND_PULLED) && pullOn(c)))
      ok = ok && waitGE(tb.sendAck, sent + 1 - (uint64_t)a.slots, sys, c);
    if (!ok) *sAbort = 1;
    if (RECV || SEND) {
      __syncthreads();
      if (*sAbort) return false;
    }
  } else {
    const uint64_t need = sent + 1 > (uint64_t)a.slots ? sent + 1 - (uint64_t)a.slots : 0;
    const bool creditWait = SEND && need > c.ackKnown;
    if (creditWait && c.tid == 32) {
      uint64_t seen = 0;
      ok = ok && waitGE(tb.sendAck, need, sys, c, seen);
      *c.sAck = seen;
    }
    if (!ok) *sAbort = 1;
    if (creditWait) {
      __syncthreads();
      if (*sAbort) return false;
      c.ackKnown = *c.sAck;
    }
  }
#if MSCCL_TRACE
  if (c.tid == 0) tr2 = globaltimer();
#endif
  const char* rslot = RECV ? tb.recvFifo + (int64_t)slotOf(recvd, (uint32_t)a.slots) * a.slotBytes : nullptr;
  char* sslot = SEND ? tb.sendFifo + (int64_t)slotOf(sent, (uint32_t)a.slots) * a.slotBytes : nullptr;
  // each protocol's data path is its own non-inlined function (separate register allocation)
  if constexpr (!ll || (!RECV && !SEND)) {
    movePiecesSimple<DT, OP, RECV, SEND, SRC, DST, REDDST>(c, tb, in, t, rslot, sslot);
#if MSCCL_WARP_FENCE
    // every warp drains its own stores before the block barrier, in parallel, so the poster's
    // fence after the barrier has (almost) nothing left to wait for
    if constexpr (SEND) {
      if (sys) fenceSys();
      else fenceGpu();
    }
#endif
  } else if constexpr (PROTO == 2) {
    if (!movePiecesLL128<DT, OP, RECV, SEND, SRC, DST, REDDST>(c, in, t, rslot, sslot, recvd + 1, sent + 1)) *sAbort = 1;
  } else {
    if (!movePiecesLL<DT, OP, RECV, SEND, SRC, DST, REDDST>(c, in, t, rslot, sslot, recvd + 1, sent + 1)) *sAbort = 1;
  }
#if MSCCL_TRACE
  if (c.tid == 0) tr3 = globaltimer();
#endif
  __syncthreads();
  if (*sAbort) return false;
#if MSCCL_TRACE
  if (c.tid == 0) tr4 = globaltimer();
#endif
  if (c.tid == 0 && ll && RECV) {  // LL/LL128: data carried its own flags; the ack frees the slot
    postFlag(tb.recvAck, recvd + 1, sys);
  } else if (c.tid == (MSCCL_POST_LAST_WARP ? c.nt - 32 : 0) && (RECV || SEND) && !ll) {
    // Simple: lane 0 of the last warp posts, so thread 0 (the head poller) goes straight to the
    // next step's wait and the fence latency overlaps it (option MSCCL_POST_LAST_WARP)
#if MSCCL_REL_STORE
    if (SEND) postRelease(tb.sendHead, sent + 1, sys);
    if (RECV) postRelease(tb.recvAck, recvd + 1, sys);
#else
    if (sys) fenceSys();
    else fenceGpu();
    if (SEND) postFlag(tb.sendHead, sent + 1, sys);
    if (RECV) postFlag(tb.recvAck, recvd + 1, sys);
#endif
  }
#if MSCCL_TRACE
  if (c.tid == 0 && a.trace) {
    uint64_t* tr = a.trace + (size_t)blockIdx.x * 8;
    uint64_t tr5 = globaltimer();
    tr[0] += tr1 - tr0;  // waiting for the incoming head
    tr[1] += tr2 - tr1;  // barrier (incl. the credit wait of thread 32)
    tr[2] += tr3 - tr2;  // thread 0's own data work
    tr[3] += tr4 - tr3;  // barrier after the data loop (slowest thread)
    tr[4] += tr5 - tr4;  // fence + flag stores
    tr[5] += 1;
  }
#endif
  if (SEND) sent++;
  if (RECV) recvd++;
  return true;
}

// ------------------------------------------------------------------ multimem ops (reading R23)
// mrd / mst / mrs address the same chunk of every rank's buffer. With NVSwitch multicast
// they are one multimem.ld_reduce / multimem.st per vector on the multicast address; this
// interpreter path is the unicast form of the same semantics: loads from every rank's copy
// (peer memory over NVLink, or the same HBM for virtual ranks), folded in ascending rank order
// with fp32 accumulation and one rounding for fp16 / bf16 sums (what the switch's .acc::f32
// reduction computes), and one store per rank.
template <int DT, int OP, int VB>
struct MMAcc {  // fold of R VB-byte vectors in ascending rank order
  typedef typename VecT<VB>::T Vec;
  static constexpr bool kHalfSum = (DT == DT_BF16 || DT == DT_F16) && OP == R_SUM;
  static constexpr int NH = VB / 2;
  float f[NH];
  Vec v;
  static __device__ __forceinline__ float widen(uint16_t x) {
    if constexpr (DT == DT_BF16) return __uint_as_float(((uint32_t)x) << 16);
    else return __half2float(__ushort_as_half(x));
  }
  static __device__ __forceinline__ uint16_t narrow(float x) {
    if constexpr (DT == DT_BF16) return __bfloat16_as_ushort(__float2bfloat16_rn(x));
    else return __half_as_ushort(__float2half_rn(x));
  }
  __device__ __forceinline__ void first(const Vec& x) {
    if constexpr (kHalfSum) {
      const uint16_t* h = reinterpret_cast<const uint16_t*>(&x);
#pragma unroll
      for (int k = 0; k < NH; k++) f[k] = widen(h[k]);
    } else {
      v = x;
    }
  }
  __device__ __forceinline__ void add(const Vec& x) {
    if constexpr (kHalfSum) {
      const uint16_t* h = reinterpret_cast<const uint16_t*>(&x);
#pragma unroll
      for (int k = 0; k < NH; k++) f[k] = f[k] + widen(h[k]);
    } else {
      v = vop<DT, OP>(v, x);
    }
  }
  __device__ __forceinline__ Vec result() const {
    if constexpr (kHalfSum) {
      Vec r;
      uint16_t* h = reinterpret_cast<uint16_t*>(&r);
#pragma unroll
      for (int k = 0; k < NH; k++) h[k] = narrow(f[k]);
      return r;
    } else {
      return v;
    }
  }
};

#ifndef MSCCL_MM_BATCH
#define MSCCL_MM_BATCH 4  // ranks whose 32-byte loads are in flight together (multimem path)
#endif

// Hardware multicast (NVLS): one multimem.ld_reduce returns the reduction of the 16 bytes at
// this address over every GPU bound to the multicast object; multimem.st writes 16 bytes to
// all of them. fp16 / bf16 sums accumulate in fp32 inside the switch (.acc::f32, reading R23).
template <int DT, int OP>
struct MCOps {
  static constexpr bool kReduce = (DT == DT_BF16 || DT == DT_F16 || DT == DT_F32) && OP == R_SUM;
  static __device__ __forceinline__ uint4 ldReduce(const char* p) {
    uint4 v;
    if constexpr (DT == DT_BF16) {
      asm volatile("multimem.ld_reduce.relaxed.sys.global.add.acc::f32.v4.bf16x2 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    } else if constexpr (DT == DT_F16) {
      asm volatile("multimem.ld_reduce.relaxed.sys.global.add.acc::f32.v4.f16x2 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    } else {
      asm volatile("multimem.ld_reduce.relaxed.sys.global.add.v4.f32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    }
    return v;
  }
  static __device__ __forceinline__ void st(char* p, const uint4& v) {  // bit pattern, any dtype
    asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y),
                 "r"(v.z), "r"(v.w) : "memory");
  }
};

// returns true when the piece was done through the multicast addresses
template <int DT, int OP, int KIND>
__device__ __forceinline__ bool multicastPiece(const Ctx& c, const DevInstr& in, int64_t so, int64_t dof, int64_t m) {
  typedef typename DType<DT>::T T;
  constexpr bool RALL = KIND != K_MST, WALL = KIND != K_MRD;
  const RankArgs& ra = *c.ra;
  const char* ms = ra.mcBuf[in.srcBuf];
  char* md = ra.mcBuf[in.dstBuf];
  if (RALL && (!MCOps<DT, OP>::kReduce || !ms)) return false;
  if (WALL && !md) return false;
  const int64_t bytes = m * (int64_t)sizeof(T);
  if ((bytes & 15) || ((so | dof) & 15)) return false;
  const int64_t nvec = bytes / 16;
  for (int64_t i = c.tid; i < nvec; i += c.nt) {
    uint4 v;
    if constexpr (RALL) v = MCOps<DT, OP>::ldReduce(ms + so + i * 16);
    else v = ldcg(c.mmBuf[ra.myRank][in.srcBuf] + so + i * 16);
    if constexpr (WALL) MCOps<DT, OP>::st(md + dof + i * 16, v);
    else stg(c.mmBuf[ra.myRank][in.dstBuf] + dof + i * 16, v);
  }
  if (c.tid == 0) atomicAdd(ra.stats + 1, 1ull);  // evidence: pieces done on the multicast path
  return true;
}

// VB = 32 when every span of the launch is 32-byte aligned (host: KernelArgs::mmVec32), else 16
template <int DT, int OP, int KIND, int VB>
__device__ __noinline__ void runMultimem(const Ctx& c, const DevInstr& in, int t) {
  typedef typename DType<DT>::T T;
  typedef typename VecT<VB>::T Vec;
  const KernelArgs& a = *c.a;
  const RankArgs& ra = *c.ra;
  constexpr bool RALL = KIND != K_MST, WALL = KIND != K_MRD;
  constexpr int B = MSCCL_MM_BATCH;
  const int R = ra.nRanks, me = ra.myRank;
  const int64_t w = sizeof(T), a0 = (int64_t)t * a.T;
  const uint64_t pol = policyEvictFirst();
  for (int j = 0; j < in.cnt; j++) {
    int64_t ss, sl, ds, dl;
    chunkSpan(a, in.srcBuf, (int64_t)in.srcOff + j, ss, sl);
    chunkSpan(a, in.dstBuf, (int64_t)in.dstOff + j, ds, dl);
    const int64_t L = sl < dl ? sl : dl;
    const int64_t m = (a0 + a.T < L ? a0 + a.T : L) - a0;
    if (m <= 0) continue;
    const int64_t so = (ss + a0) * w, dof = (ds + a0) * w;
    if (multicastPiece<DT, OP, KIND>(c, in, so, dof, m)) continue;
    uintptr_t al = (uintptr_t)so | (uintptr_t)dof;
    for (int p = 0; p < R; p++) al |= (uintptr_t)c.mmBuf[p][in.srcBuf] | (uintptr_t)c.mmBuf[p][in.dstBuf];
    const int64_t nvec = (al & (VB - 1)) ? 0 : m * w / VB;
    for (int64_t i = c.tid; i < nvec; i += c.nt) {
      MMAcc<DT, OP, VB> acc;
      if constexpr (RALL) {  // B ranks' loads in flight, folded in ascending rank order
        for (int p0 = 0; p0 < R; p0 += B) {
          Vec x[B];
#pragma unroll
          for (int u = 0; u < B; u++)
            if (p0 + u < R) ldStream(x[u], c.mmBuf[p0 + u][in.srcBuf] + so + i * VB, pol);
#pragma unroll
          for (int u = 0; u < B; u++) {
            if (p0 + u >= R) break;
            if (p0 + u == 0) acc.first(x[u]);
            else acc.add(x[u]);
          }
        }
      } else {
        Vec x;
        ldStream(x, c.mmBuf[me][in.srcBuf] + so + i * VB, pol);
        acc.first(x);
      }
      const Vec v = acc.result();
      for (int p = 0; p < R; p++)
        if (WALL || p == me) stHint(c.mmBuf[p][in.dstBuf] + dof + i * VB, v, pol);
    }
    for (int64_t e = nvec * VB / w + c.tid; e < m; e += c.nt) {  // scalar tail (ragged or unaligned)
      T v;
      if constexpr (RALL) {
        if constexpr (MMAcc<DT, OP, VB>::kHalfSum) {
          float f = MMAcc<DT, OP, VB>::widen(*(const T*)(c.mmBuf[0][in.srcBuf] + so + e * w));
          for (int p = 1; p < R; p++) f = f + MMAcc<DT, OP, VB>::widen(*(const T*)(c.mmBuf[p][in.srcBuf] + so + e * w));
          v = MMAcc<DT, OP, VB>::narrow(f);
        } else {
          v = *(const T*)(c.mmBuf[0][in.srcBuf] + so + e * w);
          for (int p = 1; p < R; p++) v = DType<DT>::op(OP, v, *(const T*)(c.mmBuf[p][in.srcBuf] + so + e * w));
        }
      } else {
        v = *(const T*)(c.mmBuf[me][in.srcBuf] + so + e * w);
      }
      for (int p = 0; p < R; p++)
        if (WALL || p == me) *(T*)(c.mmBuf[p][in.dstBuf] + dof + e * w) = v;
    }
  }
}

// Group barrier of a multimem thread block in cross-launch mode (reading R23): at its start,
// thread block b of this rank publishes {epoch, in ref, out ref} to line (start, b, me) of
// every rank and waits until every rank's line (start, b, p) here carries the same epoch,
// then resolves their buffer references; at its end it publishes (done, b, me) after a
// system-scope fence and waits for every rank's. Epoch = (program load tag, launch gen):
// equal on every rank for the same launch, never reused, compared for equality.
__device__ __forceinline__ uint64_t* mmLine(const KernelArgs& a, char* region, int kind, int b, int src, int R) {
  return (uint64_t*)(region + a.mmLineOff + ((size_t)(kind * MSCCL_MM_MAX_TB + b) * R + src) * 128);
}

__device__ __forceinline__ bool waitEq(const uint64_t* p, uint64_t v, const Ctx& c) {
  uint64_t t0 = 0;
  for (uint32_t it = 0;; it++) {
    if (ldAcquireSys(p) == v) return true;
    if ((it & 1023u) == 1023u) {
      const uint64_t now = globaltimer();
      if (t0 == 0) t0 = now;
      if (*(volatile uint32_t*)c.ra->abortFlag) return false;
      if (c.a->timeoutNs && now - t0 > c.a->timeoutNs) {
        raiseAbort(*c.a);
        return false;
      }
    }
  }
}

// returns false on watchdog / abort; every thread calls it (block-uniform)
static __device__ __noinline__ bool mmBarrier(const Ctx& c, const DevTB& tb, uint64_t gen, bool start) {
  const uint64_t epoch = ((uint64_t)tb.mmTag << 40) | ((gen + 1) & ((1ull << 40) - 1));
  const KernelArgs& a = *c.a;
  const RankArgs& ra = *c.ra;
  const int R = ra.nRanks, me = ra.myRank;
  bool ok = true;
  if (!start) {
    __syncthreads();                       // every thread's multimem stores are issued
    if (c.tid == 0) fenceSys();            // ... and visible system-wide before "done"
    __syncthreads();
  }
  if (c.tid < R && c.tid != me) {
    uint64_t* l = mmLine(a, ra.peerRegion[c.tid], start ? 0 : 1, tb.mmId, me, R);
    const uint64_t mcMask = (ra.mcBuf[0] ? 1u : 0u) | (ra.mcBuf[1] ? 2u : 0u);
    if (start) {
      stRelaxedSys(l + 1, ra.bufRef[0]);
      stRelaxedSys(l + 2, ra.bufRef[1]);
      stRelaxedSys(l + 3, mcMask);
      fenceSys();
    }
    stRelaxedSys(l, epoch);
    const uint64_t* mine = mmLine(a, ra.peerRegion[me], start ? 0 : 1, tb.mmId, c.tid, R);
    ok = waitEq(mine, epoch, c);
    if (ok && start && *(volatile const uint64_t*)(mine + 3) != mcMask) {  // NVLS buffers must be symmetric
      raiseAbort(a);
      ok = false;
    }
    if (ok && start) {
      for (int b = 0; b < 2; b++) {
        const uint64_t ref = *(volatile const uint64_t*)(mine + 1 + b);
        char* ptr = resolveRef(ra, c.tid, ref);
        if (!ptr) {  // a peer's buffer this process cannot reach: no multimem without it
          raiseAbort(a);
          ok = false;
        }
        c.mmBuf[c.tid][b] = ptr;
      }
    }
  }
  if (start && c.tid == me) {
    c.mmBuf[me][0] = ra.buf[0];
    c.mmBuf[me][1] = ra.buf[1];
  }
  return __syncthreads_and(ok) != 0;
}

template <int DT, int OP, int VB>
__device__ __forceinline__ void multimemOpV(const Ctx& c, const DevInstr& in, int t) {
  if (in.op == K_MST) runMultimem<DT, OP, K_MST, VB>(c, in, t);
  if constexpr (OP != R_COPY) {
    if (in.op == K_MRD) runMultimem<DT, OP, K_MRD, VB>(c, in, t);
    if (in.op == K_MRS) runMultimem<DT, OP, K_MRS, VB>(c, in, t);
  }
}
template <int DT, int OP>
__device__ __noinline__ void multimemOp(const Ctx& c, const DevInstr& in, int t) {
  if (c.a->mmVec32) multimemOpV<DT, OP, 32>(c, in, t);  // every span 32-byte aligned (host decides)
  else multimemOpV<DT, OP, 16>(c, in, t);
}

// MM: the kernel variant for programs with multimem ops (reading R23). Their code lives only
// in that variant: a call into it from the kernel body raised the register pressure of every
// other data path of the kernel (ptxas -v: spills in every movePieces / runOp), so programs
// without multimem ops run kernels that do not contain it.
template <int DT, int OP, int PROTO, bool MM>
__device__ __forceinline__ bool dispatch(const Ctx& c, const DevTB& tb, const DevInstr& in, int t, uint64_t& sent,
                                         uint64_t& recvd, volatile int* sAbort) {
  if constexpr (MM) {
    if (in.op >= K_MRD) {
      multimemOp<DT, OP>(c, in, t);
      __syncthreads();
      return true;
    }
  }
  switch (in.op) {  // Fig. 5 line 18; every case ends (the figure's fall-through is reading R10)
    case K_SEND: return runOp<DT, OP, PROTO, false, true, true, false, false>(c, tb, in, t, sent, recvd, sAbort);
    case K_RECV: return runOp<DT, OP, PROTO, true, false, false, true, false>(c, tb, in, t, sent, recvd, sAbort);
    case K_COPY: return runOp<DT, OP, PROTO, false, false, true, true, false>(c, tb, in, t, sent, recvd, sAbort);
    case K_RCS: return runOp<DT, OP, PROTO, true, true, false, true, false>(c, tb, in, t, sent, recvd, sAbort);

    default: break;
  }
  if (OP != R_COPY) {
    switch (in.op) {

      case K_REDUCE: return runOp<DT, OP, PROTO, false, false, true, true, true>(c, tb, in, t, sent, recvd, sAbort);
      case K_RRC: return runOp<DT, OP, PROTO, true, false, true, true, false>(c, tb, in, t, sent, recvd, sAbort);
      case K_RRS: return runOp<DT, OP, PROTO, true, true, true, false, false>(c, tb, in, t, sent, recvd, sAbort);
      case K_RRCS: return runOp<DT, OP, PROTO, true, true, true, true, false>(c, tb, in, t, sent, recvd, sAbort);
      default: break;
    }
  }
  return true;  // nop
}

// ------------------------------------------------------------------ fused local reduce chains
// A run of local instructions [cpy(src0 -> D)] re(src1 -> D) re(src2 -> D) ... on one
// destination D (marked by the loader, reading R16) is executed in ONE pass: acc = src0
// (or D), acc = acc (+) src_k in program order, one store — the same operations in the same
// order as the sequential instructions (bit-identical), without a global round trip and a
// barrier per instruction. Pieces whose members disagree on length fall back to the
// sequential instructions.
#define MSCCL_MAX_CHAIN 16
// Operand loads in flight per vector in a fused chain: 8 in the LL kernels (latency),
// 2 in the Simple and LL128 kernels (a larger batch there makes ptxas spill in their data loops,
// measured -12 % ring bandwidth).
// Operand table of one chain piece, built in shared memory by threads 0..L-1 in parallel
// (thread k resolves member k's source chunk) instead of by every thread in turn.
struct ChainSmem {
  const char* src[MSCCL_MAX_CHAIN];
  int64_t m[MSCCL_MAX_CHAIN];
  char* dst;
  int64_t dl;
};
template <int DT, int OP, int BATCH>
__device__ __noinline__ void chainExec(const Ctx& c, const DevInstr* mem, int L, int t, ChainSmem& cs) {
  typedef typename DType<DT>::T T;
  const KernelArgs& a = *c.a;
  const RankArgs& ra = *c.ra;
  const int64_t w = sizeof(T);
  const int64_t a0 = (int64_t)t * a.T;
  const bool headCopy = mem[0].op == K_COPY;
#if MSCCL_TRACE
  uint64_t ct0 = c.tid == 0 ? globaltimer() : 0, ct1 = 0, ct2 = 0;
#endif
  for (int j = 0; j < mem[0].cnt; j++) {
    if (c.tid < L) {
      const int k = c.tid;
      int64_t ds, dl, ss, sl;
      chunkSpan(a, mem[0].dstBuf, (int64_t)mem[0].dstOff + j, ds, dl);
      chunkSpan(a, mem[k].srcBuf, (int64_t)mem[k].srcOff + j, ss, sl);
      const int64_t Lk = sl < dl ? sl : dl;
      cs.m[k] = (a0 + a.T < Lk ? a0 + a.T : Lk) - a0;
      cs.src[k] = ra.buf[mem[k].srcBuf] + (ss + a0) * w;
      if (k == 0) {
        cs.dst = ra.buf[mem[0].dstBuf] + (ds + a0) * w;
        cs.dl = dl;
      }
    }
    __syncthreads();
#if MSCCL_TRACE
    if (c.tid == 0) ct1 = globaltimer();
#endif
    const int64_t m = cs.m[0];
    bool same = true;
    uintptr_t al = (uintptr_t)cs.dst;
    for (int k = 0; k < L; k++) {
      same = same && cs.m[k] == m;
      al |= (uintptr_t)cs.src[k];
    }
    char* dst = cs.dst;
    if (!same) {  // sequential fallback (a barrier between members: element->thread maps differ)
      for (int k = 0; k < L; k++) {
        const int64_t mk = cs.m[k];
        if (mk > 0) {
          if (mem[k].op == K_COPY)
            pieceSimple<DT, OP, false, false, true, true, false>(mk, nullptr, cs.src[k], dst, nullptr, c.tid, c.nt);
          else
            pieceSimple<DT, OP, false, false, true, true, true>(mk, nullptr, cs.src[k], dst, nullptr, c.tid, c.nt);
        }
        __syncthreads();
      }
      continue;
    }
    if (m > 0) {
      const int64_t bytes = m * w;
      const int64_t nvec = (al & 15) ? 0 : bytes / 16;
      // operands of a vector are loaded in batches before they are folded (in program order),
      // so a chain costs about one memory round trip per batch, not one per member
      const char* first = headCopy ? cs.src[0] : dst;
      const int k0 = headCopy ? 1 : 0;
      for (int64_t i = c.tid; i < nvec; i += c.nt) {
        uint4 acc = ldcg(first + i * 16);
        for (int kb = k0; kb < L; kb += BATCH) {
          uint4 v[BATCH];
#pragma unroll
          for (int u = 0; u < BATCH; u++)
            if (kb + u < L) v[u] = ldcg(cs.src[kb + u] + i * 16);
#pragma unroll
          for (int u = 0; u < BATCH; u++)
            if (kb + u < L) acc = vop<DT, OP>(acc, v[u]);
        }
        stg(dst + i * 16, acc);
      }
      for (int64_t e = nvec * 16 / w + c.tid; e < m; e += c.nt) {
        T acc = headCopy ? *(const T*)(cs.src[0] + e * w) : *(const T*)(dst + e * w);
        for (int k = headCopy ? 1 : 0; k < L; k++) acc = DType<DT>::op(OP, acc, *(const T*)(cs.src[k] + e * w));
        *(T*)(dst + e * w) = acc;
      }
    }
#if MSCCL_TRACE
    if (c.tid == 0) ct2 = globaltimer();
#endif
    __syncthreads();  // the operand table is rewritten for the next piece
  }
#if MSCCL_TRACE
  if (c.tid == 0 && a.trace) {  // chain phases: operand table, data (thread 0), barrier
    uint64_t* tr = a.trace + (size_t)blockIdx.x * 8;
    const uint64_t ct3 = globaltimer();
    tr[0] += ct1 - ct0;
    tr[1] += ct2 - ct1;
    tr[2] += ct3 - ct2;
    tr[7] += 1;
  }
#endif
}

// Simple-protocol kernels: the chain pass of reading R16 with its operand table in registers
// and one operand load per member (the shared-memory table and batched loads of chainExec
// below cut latency in the LL kernels, but their code in the Simple kernels cost 6 % of ring
// bandwidth through register allocation of the kernel body: measured A/B).
template <int DT, int OP>
__device__ __noinline__ void chainExecSimple(const Ctx& c, const DevInstr* mem, int L, int t) {
  typedef typename DType<DT>::T T;
  const KernelArgs& a = *c.a;
  const RankArgs& ra = *c.ra;
  const int64_t w = sizeof(T);
  const int64_t a0 = (int64_t)t * a.T;
  const bool headCopy = mem[0].op == K_COPY;
  for (int j = 0; j < mem[0].cnt; j++) {
    int64_t ds, dl;
    chunkSpan(a, mem[0].dstBuf, (int64_t)mem[0].dstOff + j, ds, dl);
    const char* srcs[MSCCL_MAX_CHAIN];
    int64_t m = -1;
    bool same = true;
    uintptr_t al = 0;
    for (int k = 0; k < L; k++) {
      int64_t ss, sl;
      chunkSpan(a, mem[k].srcBuf, (int64_t)mem[k].srcOff + j, ss, sl);
      int64_t Lk = sl < dl ? sl : dl;
      int64_t mk = (a0 + a.T < Lk ? a0 + a.T : Lk) - a0;
      if (m < 0) m = mk;
      else if (mk != m) same = false;
      srcs[k] = ra.buf[mem[k].srcBuf] + (ss + a0) * w;
      al |= (uintptr_t)srcs[k];
    }
    char* dst = ra.buf[mem[0].dstBuf] + (ds + a0) * w;
    al |= (uintptr_t)dst;
    if (!same) {  // sequential fallback (a barrier between members: element->thread maps differ)
      for (int k = 0; k < L; k++) {
        int64_t ss, sl;
        chunkSpan(a, mem[k].srcBuf, (int64_t)mem[k].srcOff + j, ss, sl);
        int64_t Lk = sl < dl ? sl : dl;
        int64_t mk = (a0 + a.T < Lk ? a0 + a.T : Lk) - a0;
        if (mk > 0) {
          if (mem[k].op == K_COPY)
            pieceSimple<DT, OP, false, false, true, true, false>(mk, nullptr, srcs[k], dst, nullptr, c.tid, c.nt);
          else
            pieceSimple<DT, OP, false, false, true, true, true>(mk, nullptr, srcs[k], dst, nullptr, c.tid, c.nt);
        }
        __syncthreads();
      }
      continue;
    }
    if (m <= 0) continue;
    const int64_t bytes = m * w;
    int64_t nvec = (al & 15) ? 0 : bytes / 16;
    for (int64_t i = c.tid; i < nvec; i += c.nt) {
      uint4 acc = headCopy ? ldcg(srcs[0] + i * 16) : ldcg(dst + i * 16);
      for (int k = headCopy ? 1 : 0; k < L; k++) acc = vop<DT, OP>(acc, ldcg(srcs[k] + i * 16));
      stg(dst + i * 16, acc);
    }
    for (int64_t e = nvec * 16 / w + c.tid; e < m; e += c.nt) {
      T acc = headCopy ? *(const T*)(srcs[0] + e * w) : *(const T*)(dst + e * w);
      for (int k = headCopy ? 1 : 0; k < L; k++) acc = DType<DT>::op(OP, acc, *(const T*)(srcs[k] + e * w));
      *(T*)(dst + e * w) = acc;
    }
  }
}


#ifndef MSCCL_MIN_BLOCKS
#define MSCCL_MIN_BLOCKS (512 / MSCCL_MAX_THREADS)
#endif
#ifndef MSCCL_SMEM_INSTR
#define MSCCL_SMEM_INSTR 64  // instructions per thread block staged in shared memory (LL / LL128)
#endif

// The LL / LL128 kernels are compiled for 1 CTA per SM: up to 255 registers, no spills (at 2 CTAs
// per SM they spilled 124 bytes in the kernel body and 130-270 bytes in the LL128 data paths).
// Latency programs use far fewer than 148 thread blocks; measured: 1 KiB one-shot LL 11.1 ->
// 10.8 us, LL128 14.0 -> 13.2 us, LL128 ring 16 MiB 113 -> 123 GB/s.
#ifndef MSCCL_LAT_MIN_BLOCKS
#define MSCCL_LAT_MIN_BLOCKS 1
#endif
#ifndef MSCCL_MM_MIN_BLOCKS
#define MSCCL_MM_MIN_BLOCKS MSCCL_MIN_BLOCKS  // multimem kernels (reading R23)
#endif
template <int DT, int OP, int PROTO, bool MM = false, int MINB = 0>  // MINB: CTAs per SM (0 = by protocol)
__global__ void __launch_bounds__(MSCCL_MAX_THREADS,
                                  MINB ? MINB : (MM ? MSCCL_MM_MIN_BLOCKS : (PROTO == 0 ? MSCCL_MIN_BLOCKS : MSCCL_LAT_MIN_BLOCKS)))
    mscclInterpreter(const __grid_constant__ KernelArgs aParam) {
  __shared__ int sAbort;
  // The launch arguments (all ranks' base pointers and tables, geometry) are copied from the
  // parameter bank into shared memory by all threads at once: every later access is a shared
  // load instead of a (serialised, on first touch) constant-cache miss.
  // (latency protocols only: kLat. The Simple kernels keep the arguments in the parameter
  // bank -- this prologue measured -6 % on the Simple ring and buys nothing at bandwidth sizes.)
  constexpr bool kLat = PROTO != 0;
  constexpr int kArgWords = kLat ? (int)(sizeof(KernelArgs) / 4) : 1;
  __shared__ __align__(16) uint32_t sArgs[kArgWords];
  if constexpr (kLat) {
    for (int i = threadIdx.x; i < kArgWords; i += blockDim.x) sArgs[i] = reinterpret_cast<const uint32_t*>(&aParam)[i];
    __syncthreads();
  }
  const KernelArgs& a = kLat ? *reinterpret_cast<const KernelArgs*>(sArgs) : aParam;
  int ls = 0;
  for (int r = 1; r < a.nLocal; r++)
    if ((int)blockIdx.x >= a.rank[r].ctaStart) ls = r;
  const int tbi = (int)blockIdx.x - a.rank[ls].ctaStart;
  const RankArgs& ra = a.rank[ls];
  if (tbi >= ra.nTB) return;
  // Prologue: the thread block's descriptor and instruction list are staged in
  // shared memory by parallel 16-byte loads, so the instruction loop never waits on a global
  // round trip to decode a step. Latency kernels load both in ONE round trip from the
  // program's per-block record (DevTB followed by its instructions); the generation word is
  // loaded at the same time.
  __shared__ __align__(16) DevTB sTB;
  __shared__ __align__(16) DevInstr sIns[kLat ? MSCCL_SMEM_INSTR : 1];
  uint64_t genEarly = 0;
  const DevInstr* ins = nullptr;
  if constexpr (kLat) {
    if (ra.tbRecStride) {
      const uint4* rec = reinterpret_cast<const uint4*>(ra.tbRec + (int64_t)tbi * ra.tbRecStride);
      const int nw = (int)(ra.tbRecStride / 16), ntb = (int)(sizeof(DevTB) / 16);
      for (int i = threadIdx.x; i < nw; i += blockDim.x) {
        const uint4 v = rec[i];
        if (i < ntb) reinterpret_cast<uint4*>(&sTB)[i] = v;
        else reinterpret_cast<uint4*>(sIns)[i - ntb] = v;
      }
      genEarly = *(volatile uint64_t*)&ra.gen[tbi];
      ins = sIns;
    } else if (threadIdx.x < sizeof(DevTB) / 16) {
      reinterpret_cast<uint4*>(&sTB)[threadIdx.x] = reinterpret_cast<const uint4*>(&ra.tbs[tbi])[threadIdx.x];
    }
    __syncthreads();
  }
  const DevTB& tb = kLat ? sTB : ra.tbs[tbi];
  if (!ins) {
    ins = ra.instrs + tb.instrStart;
    if (kLat && tb.nSteps <= MSCCL_SMEM_INSTR) {
      for (int i = threadIdx.x; i < tb.nSteps * (int)(sizeof(DevInstr) / 16); i += blockDim.x)
        reinterpret_cast<uint4*>(sIns)[i] = reinterpret_cast<const uint4*>(ins)[i];
      ins = sIns;
    }
  }
  __shared__ uint64_t sAck;
  __shared__ char* sPeerDst[3];
  __shared__ char* sMM[MSCCL_MM_MAX_RANKS][2];
  __shared__ ChainSmem sChain;
  Ctx c{&a, &ra, (int)threadIdx.x, (int)blockDim.x, 0, &sAck, sPeerDst, false, 0, sMM};
  if (MM && a.mm == 1 && (int)threadIdx.x < a.nLocal) {  // every rank in this launch: slot r = rank r
    sMM[threadIdx.x][0] = a.rank[threadIdx.x].buf[0];
    sMM[threadIdx.x][1] = a.rank[threadIdx.x].buf[1];
  }
  if (threadIdx.x == 0) {
    sAbort = 0;
    // one-launch direct placement: the send peer is local rank tb.sendPeer of this launch
    for (int b = 0; b < 3; b++)
      sPeerDst[b] = (a.direct == 1 && tb.sendPeer >= 0) ? a.rank[tb.sendPeer].buf[b] : nullptr;
  }
  uint64_t sent = tb.sendFifo ? *(volatile uint64_t*)tb.sendCnt : 0;
  uint64_t recvd = tb.recvFifo ? *(volatile uint64_t*)tb.recvCnt : 0;
  const uint64_t gen = (kLat && ra.tbRecStride) ? genEarly : *(volatile uint64_t*)&ra.gen[tbi];
  // Launch ordinals per connection (word 1 of the persistent counter lines) stay in lock-step
  // on both ends in every launch; in cross-launch direct mode the receiving thread block also
  // publishes where its destinations are (reading R15b), released by one fence.
  if (threadIdx.x == 32 && tb.sendFifo) {
    c.sendL = *(volatile uint64_t*)(tb.sendCnt + 1) + 1;
    *(volatile uint64_t*)(tb.sendCnt + 1) = c.sendL;
  }
  if (threadIdx.x == 0 && tb.recvFifo) {
    const uint64_t L = *(volatile uint64_t*)(tb.recvCnt + 1) + 1;
    *(volatile uint64_t*)(tb.recvCnt + 1) = L;
    if (a.direct == 2) {
      for (int b = 0; b < 4; b++)  // in / out / scratch refs, then the tile size (R19 check)
        postFlag(tb.recvReady + 1 + b, b < 3 ? ra.bufRef[b] : (uint64_t)a.T, a.sysScope != 0);
      if (a.sysScope) fenceSys();
      else fenceGpu();
      postFlag(tb.recvReady, L, a.sysScope != 0);
    }
  }
  // semaphore posts (fence + store) by lane 0 of the last warp: thread 0 polls the next step's
  // head / dependencies meanwhile; every post follows a block barrier (option MSCCL_POST_LAST_WARP)
  const int kPoster = MSCCL_POST_LAST_WARP ? (int)blockDim.x - 32 : 0;
  __syncthreads();
  if constexpr (MM) {
    if (a.mm == 2 && tb.mmId >= 0 && !mmBarrier(c, tb, gen, true)) return;
  }
  for (int t = 0; t < a.I; t++) {
    for (int s = 0; s < tb.nSteps; s++) {
      const DevInstr in = ins[s];
      if constexpr (OP != R_COPY) {
        if (in.flags & DI_CHAIN_HEAD) {  // reading R16: fused local reduce chain
          const int L = in.chainLen;
          bool ok = true;
          if constexpr (PROTO == 0) {
            for (int k = 0; k < L && ok; k++) {  // all members' dependencies first
              const DevInstr& mk = ins[s + k];
              for (int d = c.tid; d < mk.nDeps && ok; d += c.nt) ok = waitDep(ra, ra.deps[mk.depStart + d], gen, t, c);
            }
          } else {
            // flattened dependency f goes to thread f mod nt; a thread first collects its
            // dependency words, then waits on all of them, so the waits of different members
            // overlap (waiting inside the member loop serialises them: one member per loop trip)
            constexpr int KD = 4;
            uint64_t mine[KD];
            int nm = 0;
            for (int k = 0, base = 0; k < L; k++) {
              const DevInstr& mk = ins[s + k];
              for (int d = ((c.tid - base) % c.nt + c.nt) % c.nt; d < mk.nDeps; d += c.nt) {
                const uint64_t dw = ra.deps[mk.depStart + d];
                if (nm < KD) mine[nm++] = dw;
                else ok = ok && waitDep(ra, dw, gen, t, c);  // more than KD per thread: in order
              }
              base += mk.nDeps;
            }
#pragma unroll
            for (int i = 0; i < KD; i++)
              if (i < nm) ok = ok && waitDep(ra, mine[i], gen, t, c);
          }
          if (!ok) sAbort = 1;
          __syncthreads();
          if (sAbort) return;
          if constexpr (PROTO == 0) chainExecSimple<DT, OP>(c, ins + s, L, t);
          else chainExec<DT, OP, PROTO == 1 ? 8 : 2>(c, ins + s, L, t, sChain);
          __syncthreads();
          s += L - 1;
          if (ins[s].hasDep && c.tid == kPoster) {
            fenceGpu();
            stRelaxedGpu(&ra.sem[tbi], (gen << 40) | ((uint64_t)t * (uint64_t)tb.nSteps + (uint64_t)s + 1));
          }
          continue;
        }
      }
      if (in.nDeps) {  // Fig. 5 lines 15-16; barrier after the waits (reading R10)
        bool ok = true;
        for (int d = c.tid; d < in.nDeps && ok; d += c.nt) ok = waitDep(ra, ra.deps[in.depStart + d], gen, t, c);
        if (!ok) sAbort = 1;
        __syncthreads();
        if (sAbort) return;
      }
      if (!dispatch<DT, OP, PROTO, MM>(c, tb, in, t, sent, recvd, &sAbort)) return;
      if (in.hasDep) {  // Fig. 5 lines 25-27: the step is complete before the semaphore moves
        if (c.tid == kPoster) {
          fenceGpu();
          stRelaxedGpu(&ra.sem[tbi], (gen << 40) | ((uint64_t)t * (uint64_t)tb.nSteps + (uint64_t)s + 1));
        }
      }
    }
  }
  if constexpr (MM) {
    if (a.mm == 2 && tb.mmId >= 0 && !mmBarrier(c, tb, gen, false)) return;
  }
  if (threadIdx.x == 0) {  // epilogue: persist the connection counters and the generation
    if (tb.sendFifo) *(volatile uint64_t*)tb.sendCnt = sent;
    if (tb.recvFifo) *(volatile uint64_t*)tb.recvCnt = recvd;
    *(volatile uint64_t*)&ra.gen[tbi] = gen + 1;
  }
}

}  // namespace msccl
