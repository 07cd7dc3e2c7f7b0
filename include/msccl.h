/*
 * msccl.h — C ABI of the B200-native MSCCL-IR interpreter (libmsccl_b200.so).
 *
 * The runtime "is API-compatible with NCCL allowing existing ML workloads to easily
 * convert" (MSCCLang, ASPLOS '23, §1): entry points, enum values and argument
 * order mirror nccl.h (2.28). A collective call selects a loaded MSCCL-IR program by
 * "user configurable size ranges" (§6) and runs it in ONE persistent CUDA
 * kernel per GPU that interprets the program's instruction lists (§6.2, Fig. 5
 * P:L1281-1310). Unlike the paper's runtime there is no NCCL fallback: a call with no
 * matching program returns mscclNoMatchingProgram and launches nothing.
 *
 * Conventions for every function:
 *  - returns mscclResult_t; never throws, never aborts the process;
 *  - pointers named *buff are DEVICE pointers on the communicator's device, caller-owned,
 *    valid until the stream reaches the operation; `count`s are ELEMENTS of `datatype`;
 *  - a communicator is not thread-safe (NCCL rule); all ranks must load the same programs
 *    in the same order and issue the same collectives with the same count/dtype/op;
 *  - calls are asynchronous on `stream` and contain no host synchronisation. A call
 *    allocates only when a program loaded WITHOUT maxBytes needs more scratch than any
 *    earlier call (it then grows; the old buffer lives until unload). Programs loaded with
 *    maxBytes pre-size their scratch, so every call in their size range can be captured in
 *    a CUDA graph, the first one included; a call that would have to grow scratch while the
 *    stream is capturing returns mscclInvalidUsage instead;
 *  - mscclGetLastError(comm) returns a human-readable reason for the last failure
 *    (for program errors: rank/thread block/step and the violated rule V1..V9).
 */
#ifndef MSCCL_B200_H_
#define MSCCL_B200_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct mscclComm* mscclComm_t;
typedef struct mscclProgram* mscclProgram_t;
typedef struct CUstream_st* mscclStream_t; /* == cudaStream_t */

/* 0..7 are numerically identical to ncclResult_t. */
typedef enum {
  mscclSuccess = 0,
  mscclUnhandledCudaError = 1,
  mscclSystemError = 2,
  mscclInternalError = 3,
  mscclInvalidArgument = 4,
  mscclInvalidUsage = 5,
  mscclRemoteError = 6,       /* watchdog timeout / peer abort (sticky, async) */
  mscclInProgress = 7,
  mscclInvalidProgram = 8,    /* IR failed to parse or validate */
  mscclNoMatchingProgram = 9  /* no loaded program for (collective, nranks, bytes) */
} mscclResult_t;

/* Numerically identical to ncclDataType_t. */
typedef enum {
  mscclInt8 = 0, mscclUint8 = 1, mscclInt32 = 2, mscclUint32 = 3, mscclInt64 = 4,
  mscclUint64 = 5, mscclFloat16 = 6, mscclFloat32 = 7, mscclFloat64 = 8, mscclBfloat16 = 9,
  mscclNumTypes = 10
} mscclDataType_t;

/* Numerically identical to ncclRedOp_t; ncclAvg (4) is rejected (InvalidArgument). */
typedef enum { mscclSum = 0, mscclProd = 1, mscclMax = 2, mscclMin = 3, mscclNumOps = 4 } mscclRedOp_t;

/* Size of the opaque handle written by mscclCommExportHandle. */
#define MSCCL_HANDLE_BYTES 128

/* ---------------------------------------------------------------- communicators */

/* One process drives `ndev` ranks; rank i runs on device devlist[i] (devlist may be NULL:
 * devices 0..ndev-1). Distinct devices are connected by CUDA peer access over NVLink.
 * Repeated device ids are VIRTUAL RANKS (at most 8 per device): several ranks on one GPU, whose buffers and
 * FIFOs all live in that GPU's HBM (used for correctness work on one GPU). Ranks that
 * share a device must issue their calls inside mscclGroupStart/End so that they run in
 * ONE cooperative launch (all thread blocks co-resident, §6.2).
 * comms[ndev] is written; each must be destroyed with mscclCommDestroy. */
mscclResult_t mscclCommInitAll(mscclComm_t* comms, int ndev, const int* devlist);

/* One process per GPU: allocate this rank's shared region (FIFOs, flags) on cudaDev.
 * Then mscclCommExportHandle -> exchange (e.g. torch.distributed all_gather) ->
 * mscclCommConnect before the first collective. */
mscclResult_t mscclCommInitRank(mscclComm_t* comm, int nranks, int rank, int cudaDev);

/* Writes MSCCL_HANDLE_BYTES bytes (CUDA IPC handle of the shared region) to `handle`;
 * *bytes (if not NULL) receives MSCCL_HANDLE_BYTES. */
mscclResult_t mscclCommExportHandle(mscclComm_t comm, void* handle, size_t* bytes);

/* allHandles: nranks * MSCCL_HANDLE_BYTES bytes, rank order. Opens every peer's region. */
mscclResult_t mscclCommConnect(mscclComm_t comm, const void* allHandles);

/* Frees the region, programs and IPC mappings (synchronises the device). */
mscclResult_t mscclCommDestroy(mscclComm_t comm);

mscclResult_t mscclCommCount(const mscclComm_t comm, int* count);

/* Counters of this rank (synchronises with the device to read them), up to n of:
 * [0] cross-launch ready handshakes in which a sender of this rank found a reachable
 *     destination and stored directly into a peer (device-side count, reading R15b);
 * [1] launches with one-launch direct placement (every rank in the launch, reading R15);
 * [2] launches in which this rank published a reachable destination (cross-launch mode);
 * [3] multimem pieces executed through an NVSwitch multicast address (device-side count);
 * [4] V9 re-checks run at a launch's real pipeline depth (one per program and depth I > 2). */
mscclResult_t mscclCommGetStats(mscclComm_t comm, int64_t* stats, int n);
mscclResult_t mscclCommUserRank(const mscclComm_t comm, int* rank);
mscclResult_t mscclCommCuDevice(const mscclComm_t comm, int* device);

/* Sticky asynchronous error: mscclRemoteError after a device watchdog timeout (a spin
 * wait exceeded MSCCL_TIMEOUT_S, default 60 s; <= 0 disables the watchdog) or an abort
 * raised by a peer. */
mscclResult_t mscclCommGetAsyncError(mscclComm_t comm, mscclResult_t* asyncError);

/* ---------------------------------------------------------------- buffer registration
 * Direct placement (readings R15 / R15b; the paper's future work, §7.5
 * P:L2615-2624): a sender stores a message straight into the receiver's destination chunk
 * instead of the receiver-side FIFO. Within one process (mscclCommInitAll, any devices)
 * every buffer is reachable and nothing needs registering. For one process per GPU (CUDA
 * IPC), a receiver's buffer is reachable only if it lies inside a REGISTERED range:
 *   mscclCommRegister(comm, buff, size, &reg)   every rank, same order (collective)
 *   mscclRegExport(reg, desc)                   MSCCL_REG_DESC_BYTES bytes
 *   (exchange the descriptors, e.g. torch.distributed all_gather)
 *   mscclRegConnect(reg, allDescs)              nranks * MSCCL_REG_DESC_BYTES, rank order;
 *                                               maps every peer's range; all ranks must
 *                                               return from it before any uses the buffer
 * A call whose recvbuff (or sendbuff, for in-place programs) is not inside a connected
 * registration simply uses the FIFO for messages to this rank. Option (reading R19b,
 * MSCCL_DIRECT_TILE=2): a program whose every message is a direct placement and that forwards
 * nothing (e.g. the direct AllToAll) moves each chunk as ONE message when this rank's sendbuff
 * and recvbuff are both registered; every rank must then have registered its buffers for the
 * call, otherwise the ranks disagree on the message size and the launch ends in
 * mscclRemoteError (checked on the per-launch ready line), never in a store past a FIFO slot. Registration allocates and
 * synchronises (not capturable). mscclCommDeregister unmaps (collective, after the stream
 * work that used the buffer has completed). Errors: InvalidArgument (null, size 0, range
 * not inside one device allocation, more than MSCCL_MAX_REGISTRATIONS), UnhandledCudaError. */
typedef struct mscclReg* mscclReg_t;
#define MSCCL_REG_DESC_BYTES 128
mscclResult_t mscclCommRegister(mscclComm_t comm, void* buff, size_t size, mscclReg_t* reg);
mscclResult_t mscclRegExport(mscclReg_t reg, void* desc);
mscclResult_t mscclRegConnect(mscclReg_t reg, const void* allDescs);
mscclResult_t mscclCommDeregister(mscclComm_t comm, mscclReg_t reg);

/* ---------------------------------------------------------------- NVLS buffers
 * NVSwitch multicast (reading R23). mscclNvlsAlloc allocates
 * `bytes` on every rank's GPU of one single-process communicator set (mscclCommInitAll, one
 * rank per distinct device, comms in rank order), binds all of them to one multicast
 * object, and writes each rank's (unicast) pointer to ptrs[rank]. A multimem program whose
 * sendbuff / recvbuff lie inside such a buffer (at the same offset on every rank) runs its
 * mrd / mst / mrs instructions as multimem.ld_reduce / multimem.st on the multicast address
 * (fp16 / bf16 / fp32 sums, and stores of any type; other dtype / op pairs and buffers
 * outside NVLS buffers use the unicast form). Not capturable (allocates). Errors:
 * InvalidArgument (not a full rank-ordered clique), InvalidUsage (two ranks on one device),
 * SystemError (no multicast support), UnhandledCudaError. mscclNvlsSupported reports
 * CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED of a device (0 when the driver lacks the API). */
mscclResult_t mscclNvlsSupported(int cudaDev, int* supported);
mscclResult_t mscclNvlsAlloc(mscclComm_t* comms, int ncomms, size_t bytes, void** ptrs);
mscclResult_t mscclNvlsFree(mscclComm_t* comms, int ncomms, void** ptrs);

/* ---------------------------------------------------------------- programs */

/* Parse + validate an MSCCL-IR program (text, irBytes bytes; copied) and upload its
 * instruction tables for this rank (§6.2 "Initialization"). The program is
 * selected for calls whose byte size (count * element size of the call's datatype) is
 * in [minBytes, maxBytes); maxBytes == 0 means unbounded. First loaded program wins.
 * Errors: mscclInvalidProgram (parse/validation, see mscclGetLastError). */
mscclResult_t mscclLoadProgram(mscclComm_t comm, const char* ir, size_t irBytes, size_t minBytes,
                               size_t maxBytes, mscclProgram_t* program);
mscclResult_t mscclUnloadProgram(mscclComm_t comm, mscclProgram_t program);

/* Statistics of a loaded program for this rank: thread blocks (= CTAs launched), total
 * instructions, and whether it is in place. Any pointer may be NULL. */
mscclResult_t mscclProgramInfo(mscclProgram_t program, int* nThreadBlocks, int* nInstructions, int* inplace);

/* Algorithmic memory traffic of this rank's program, in chunk-sized touches per pipeline
 * pass (bytes per launch = touches * chunk bytes): each instruction reads/writes its
 * operands once per chunk — send 2, recv 2, copy 2, reduce 3, rrc 3, rrs 3, rrcs 4, rcs 3 —
 * and with direct placement (directPlacement != 0, reading R15) a direct recv costs 0 and
 * a direct rcs 2 (the data arrived in dst); with every rank in one launch (directPlacement
 * == 1; 2 = cross-launch) and MSCCL_DIRECT_HINTS bit 4, a pulled send costs 0 (reading R30:
 * its receive reads the input chunk instead of the FIFO slot, same count). */
mscclResult_t mscclProgramTouches(mscclProgram_t program, int directPlacement, int64_t* touches);

/* Direct-placement marking the loader computes for rank `rank` of an IR program (reading
 * R15; needs no GPU). For every instruction in (thread block, step) order of that rank,
 * flags[k] = bit 0 DIRECT_SEND (the message is stored into the receiver's destination),
 * bit 1 DIRECT_RECV (the data is already in dst when the head arrives), bit 2 PULLED_RECV (the
 * receive reads the sender's input chunk itself, reading R30), bit 3 PULLED_SEND (its
 * partner: moves no data); for a direct send
 * rdst[2k], rdst[2k+1] = the receiver's destination buffer (0 i, 1 o, 2 s) and chunk.
 * maxInstr = capacity of flags (rdst: 2*maxInstr); *nInstr = instructions of the rank.
 * Exported so the CPU oracle's race detector (oracle/races.py) can check the marking
 * independently. Returns mscclInvalidProgram if the IR does not parse or validate. */
mscclResult_t mscclDebugDirectPlacement(const char* ir, size_t irBytes, int rank, int32_t* flags,
                                        int32_t* rdst, int maxInstr, int* nInstr);

/* Test hook: set the launch generation of every thread block of `program` (the counter the
 * dependency semaphores carry, reading R4), so tests can cross the 2^24-launch wrap of the
 * semaphores' generation field without 16 M launches. Synchronises the device. */
mscclResult_t mscclDebugSetGeneration(mscclProgram_t program, uint64_t generation);

/* Comm-free structural validation (rules V1..V9 of DESIGN.md) — needs no GPU.
 * slots = FIFO slots per connection used by the deadlock check (0 = library default),
 * maxThreadBlocks = co-residency limit per rank (0 = 148). err (may be NULL) receives a
 * NUL-terminated reason. Returns mscclSuccess or mscclInvalidProgram. */
mscclResult_t mscclValidateProgram(const char* ir, size_t irBytes, int nranks, int slots,
                                   int maxThreadBlocks, char* err, size_t errBytes);

/* ---------------------------------------------------------------- collectives
 * Semantics (n = count / per-rank block):
 *   AllReduce     out_r[e]       = (op)_q in_q[e]
 *   AllGather     out_r[q*n + e] = in_q[e]                          (sendcount = n)
 *   ReduceScatter out_r[e]       = (op)_q in_q[r*n + e]             (recvcount = n)
 *   AllToAll      out_r[q*n + e] = in_q[r*n + e]   (count per peer)
 * In place (NCCL forms): AllReduce sendbuff == recvbuff; AllGather sendbuff ==
 * recvbuff + rank*n; ReduceScatter recvbuff == sendbuff + rank*n. An in-place program
 * called out of place gets a device copy send->recv first; an out-of-place program
 * called in place must be marked aliassafe in its IR, else mscclInvalidUsage.
 * count == 0 is a no-op. Floating-point results are bit-identical to the CPU oracle
 * executing the same program (one rounding per reduce instruction). */
mscclResult_t mscclAllReduce(const void* sendbuff, void* recvbuff, size_t count, mscclDataType_t datatype,
                             mscclRedOp_t op, mscclComm_t comm, mscclStream_t stream);
mscclResult_t mscclAllGather(const void* sendbuff, void* recvbuff, size_t sendcount, mscclDataType_t datatype,
                             mscclComm_t comm, mscclStream_t stream);
mscclResult_t mscclReduceScatter(const void* sendbuff, void* recvbuff, size_t recvcount,
                                 mscclDataType_t datatype, mscclRedOp_t op, mscclComm_t comm,
                                 mscclStream_t stream);
mscclResult_t mscclAllToAll(const void* sendbuff, void* recvbuff, size_t count, mscclDataType_t datatype,
                            mscclComm_t comm, mscclStream_t stream);

/* Run a specific loaded program regardless of size ranges (bench / tests). `count` is
 * interpreted per the program's collective as above. */
mscclResult_t mscclRunProgram(mscclProgram_t program, const void* sendbuff, void* recvbuff, size_t count,
                              mscclDataType_t datatype, mscclRedOp_t op, mscclComm_t comm, mscclStream_t stream);

/* Group semantics (ncclGroupStart/End): calls between them are recorded and launched at
 * mscclGroupEnd, one cooperative kernel per device covering every rank on that device. */
mscclResult_t mscclGroupStart(void);
mscclResult_t mscclGroupEnd(void);

/* ---------------------------------------------------------------- misc */
const char* mscclGetErrorString(mscclResult_t result);
const char* mscclGetLastError(mscclComm_t comm); /* comm may be NULL: last global error */

/* Tuning knobs (process-wide, read when a communicator is created; env vars of the same
 * name override at first use). Defaults are the tuned configuration of DESIGN.md §7:
 * "MSCCL_SLOTS" FIFO slots per connection (1..16, default 4); "MSCCL_SLOT_BYTES" Simple
 * slot (default 262144), "MSCCL_LL_SLOT_BYTES" (65536), "MSCCL_LL128_SLOT_BYTES" (262144)
 * -- each protocol has its own slots; "MSCCL_MAX_CHANNELS" (32); "MSCCL_THREADS" threads
 * per CTA (64..256, default 256: 2 CTAs per SM for Simple programs, 1 for LL / LL128, so a
 * launch holds at most 296 / 148 thread blocks); "MSCCL_TIMEOUT_S" watchdog (default 60,
 * <= 0 disables); "MSCCL_DIRECT" direct placement (1); "MSCCL_DIRECT_TILE" one tile per
 * chunk when every message is direct (1; 2 = also across processes, see registration); "MSCCL_DIRECT_HINTS" L2 hints of direct stores, a
 * bit set (default 25: bit 0 terminal direct sends evict_first, bit 3 forwarded direct sends
 * evict_normal, bit 4 pulled messages: with every rank in one launch a receive whose message
 * is a plain send of an input chunk reads that chunk itself, reading R30; bit 1 demote
 * forwarded lines after reading, bit 2 FIFO stores evict_normal: measured slower, off);
 * "MSCCL_MAX_REGISTRATIONS" (64). All ranks must
 * use the same values (mscclCommConnect checks). Returns mscclInvalidArgument for an
 * unknown key. */
mscclResult_t mscclSetParam(const char* key, int64_t value);
mscclResult_t mscclGetParam(const char* key, int64_t* value);

/* Number of interpreter kernels this process has launched (for launch accounting). */
uint64_t mscclLaunchCount(void);

#ifdef __cplusplus
}
#endif
#endif /* MSCCL_B200_H_ */
