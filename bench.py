#!/usr/bin/env python3
"""Benchmark of the MSCCL-IR interpreter (MSCCLang, ASPLOS '23) on B200.

Metric (BASELINE.json): AllReduce / AllToAll bus bandwidth vs size at 2/4/8 B200 and the
1 KB latency. busBW follows the nccl-tests convention: algBW x 2(R-1)/R for
AllReduce and x (R-1)/R for AllGather / ReduceScatter / AllToAll, with S = bytes per rank.

Default run (N = 1: one GPU, no flags) -- one JSON line:
  workload = the largest single-GPU analogue of BASELINE configs[1] ("Ring AllReduce
  8xB200, bf16, pipelined chunks"): ring AllReduce MSCCL-IR, bf16, R = 8 VIRTUAL ranks on
  one B200 (every rank's buffers, FIFOs and peer stores in that GPU's HBM, one cooperative
  interpreter launch per step), 256 MiB per rank, 1 channel x 32 instances (256 CTAs).
  One GPU cannot host NVLink traffic, so this line is HBM-bound and its roofline is the
  measured HBM copy bandwidth. Inputs: 2 GiB > 126 MB L2, no flush needed.
  Extras measured on the same virtual ranks (each named by the BASELINE config it
  mirrors): the 1 KiB fp16 latency (configs[2]), the launch-latency floor, the AllToAll at
  256 MiB per rank (configs[3]), and AllGather / ReduceScatter (configs[4]).

Under torchrun (N > 1) each process drives one GPU as one rank over CUDA IPC peer memory
(NVLink / NVSwitch). User buffers are registered (mscclCommRegister), so messages are
placed directly into the peer's buffer (reading R15b). value = ring AllReduce busBW at S
per rank from the max over ranks of the CUDA-event time; roofline = NVLink per direction
(measured peer copy, nominal 900 GB/s); NCCL 2.28.9 runs in the same loop as the
comparison arm. MSCCL_FORCE_DEVICE=<d> puts every rank on GPU d, which exercises the
multi-process plumbing on a one-GPU box (NCCL is then skipped: it refuses two ranks on one
GPU; processes whose kernels spin on each other while time-slicing one GPU can raise Xid 109
on this driver, B200_PROFILING.md -- a plumbing check, not a measurement).

--sweep PATH : per-size JSON lines (1 KiB..1 GiB, x2) for AllReduce and AllToAll, eager and
  CUDA graph, the paper's protocol (20 warm-up + 50 timed ops) plus a
  1000-iteration latency mode for <= 64 KiB; MSCCL (size-range program sets, §6
  P:L1268-1273) and, with N > 1, NCCL.
--impl reference : the CPU oracle (oracle/sim.py) executing the same IR on a bounded
  sample of the same workload, on the host cores (the reference arm).
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

MIB = 1 << 20
SEED_SAMPLES = 4096
NVLINK_NOMINAL = 900.0  # GB/s per direction per GPU (NVLink 5)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="msccl", choices=["msccl", "reference"])
    ap.add_argument("--ranks", type=int, default=8, help="virtual ranks when N=1")
    ap.add_argument("--size-mib", type=float, default=256.0, help="bytes per rank (MiB)")
    ap.add_argument("--program", default="ring",
                    choices=["ring", "allpairs", "oneshot", "alltoall", "allgather", "allgather_direct", "reducescatter",
                             "nvls"])
    ap.add_argument("--channels", type=int, default=1)
    ap.add_argument("--split", action="store_true", help="ring: AllGather half on its own channels (reading R26)")
    ap.add_argument("--rings", type=int, default=1, help="ring: K interleaved logical rings per thread block (R27)")
    ap.add_argument("--instances", type=int, default=32)
    ap.add_argument("--protocol", default="Simple")
    ap.add_argument("--threads", type=int, default=256)
    ap.add_argument("--slots", type=int, default=4)
    ap.add_argument("--slot-kib", type=int, default=256)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-nccl", action="store_true")
    ap.add_argument("--no-register", action="store_true", help="N>1: do not register buffers (FIFO only)")
    ap.add_argument("--quiet-extra", action="store_true", help="skip the extras")
    ap.add_argument("--sweep", default=None, help="write per-size JSON lines to this path (and stdout)")
    ap.add_argument("--sweep-max-mib", type=int, default=1024)
    return ap.parse_args()


# ----------------------------------------------------------------------------- helpers
def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def l2_peak():
    """Measured L2-resident copy throughput (tools/l2bw.cu), committed under profiles/."""
    p = os.path.join(ROOT, "profiles", "l2_peak.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["l2_gbs"]), "measured (profiles/l2_peak.json: %s)" % d.get("how", "")
    except Exception:
        return None, "unmeasured"


def ncu_traffic():
    """dram read+write bytes per launch of the interpreter, from the committed ncu summary."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get("dram_bytes_per_launch"), d
    except Exception:
        return None, None


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index=0):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,power.draw,"
                 "clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
                 "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
                 "clocks_event_reasons.sw_power_cap", "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm_, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(nm_)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


def busbw(coll, S, t, R):
    f = 2.0 * (R - 1) / R if coll == "allreduce" else (R - 1) / R
    return S / t * f / 1e9


def build_program(args, R):
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    if args.program == "ring":
        return P.ring_allreduce(R, channels=args.channels, instances=args.instances, protocol=args.protocol,
                                split_phases=args.split, rings=args.rings)
    if args.program == "allpairs":
        return P.allpairs_allreduce(R, instances=args.instances, protocol=args.protocol)
    if args.program == "oneshot":
        return P.oneshot_allreduce(R, instances=args.instances, protocol=args.protocol)
    if args.program == "nvls":
        return P.nvls_allreduce(R, args.instances)
    if args.program == "allgather":
        return P.ring_allgather(R, args.channels, args.instances, protocol=args.protocol)
    if args.program == "allgather_direct":
        return P.allpairs_allgather(R, args.instances, protocol=args.protocol)
    if args.program == "reducescatter":
        return P.ring_reducescatter(R, args.channels, args.instances, protocol=args.protocol)
    return P.alltoall_twostep(1, R, instances=args.instances, protocol=args.protocol)


def coll_of(program):
    return {"alltoall": "alltoall", "allgather": "allgather", "allgather_direct": "allgather",
            "reducescatter": "reducescatter"}.get(program,
                                                                                                  "allreduce")


def shapes(coll, n, W):
    """(send elems, recv elems, count) for S = n elements per rank (S = the larger buffer)."""
    if coll == "allgather":
        return n // W, n, n // W
    if coll == "reducescatter":
        return n, n // W, n // W
    if coll == "alltoall":
        return n, n, n // W
    return n, n, n


def nop_ir(R):
    """The smallest MSCCL-IR program: every rank one thread block with one nop. Its CUDA-graph
    replay time is the interpreter's launch-latency floor (cooperative launch + prologue +
    epilogue), against which the 1 KiB latencies are read."""
    g = "".join('<gpu id="%d" i_chunks="1" o_chunks="1" s_chunks="0"><tb id="0" send="-1" recv="-1" chan="0">'
                '<step s="0" type="nop" srcbuf="-" srcoff="-1" dstbuf="-" dstoff="-1" cnt="1" depid="-1" '
                'deps="-1" hasdep="0"/></tb></gpu>' % q for q in range(R))
    return '<algo name="nop" coll="custom" ngpus="%d" proto="LL" inplace="0" nchannels="1">%s</algo>' % (R, g)


def hop_ir(R, proto="LL"):
    """One message hop: rank r sends its chunk to rank r+1 (AllToNext without the cross-node
    relay, §7.4). Its latency minus the launch floor is the cost of one hop of the
    protocol; the 1 KiB breakdown in DESIGN.md §7 reads the one-shot and ring latencies
    against floor + hops."""
    g = []
    for q in range(R):
        tbs = []
        if q + 1 < R:
            tbs.append('<tb id="%d" send="%d" recv="-1" chan="0"><step s="0" type="s" srcbuf="i" srcoff="0" '
                       'dstbuf="-" dstoff="-1" cnt="1" depid="-1" deps="-1" hasdep="0"/></tb>' % (len(tbs), q + 1))
        if q > 0:
            tbs.append('<tb id="%d" send="-1" recv="%d" chan="0"><step s="0" type="r" srcbuf="-" srcoff="-1" '
                       'dstbuf="o" dstoff="0" cnt="1" depid="-1" deps="-1" hasdep="0"/></tb>' % (len(tbs), q - 1))
        g.append('<gpu id="%d" i_chunks="1" o_chunks="1" s_chunks="0">%s</gpu>' % (q, "".join(tbs)))
    return '<algo name="hop" coll="custom" ngpus="%d" proto="%s" inplace="0" nchannels="1">%s</algo>' % (
        R, proto, "".join(g))


def host_threads():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count()


# ----------------------------------------------------------------------------- CPU oracle
def cpu_oracle_run(R, algo, sample_bytes, reps=5):
    """Time oracle.sim.simulate on a bounded sample (same program, same dtype, same R);
    median of `reps` runs, numpy in one Python thread."""
    import numpy as np
    import synth
    from oracle import irparse, sim
    dtype = "bfloat16"
    n = int(sample_bytes // 2)
    al = irparse.parse(algo.to_xml())
    xs = [synth.hashed_numpy(q, np.arange(n), dtype) for q in range(R)]
    times = []
    for _ in range(reps):
        t0 = time.perf_counter()
        sim.simulate(al, xs, n, dtype, "sum")
        times.append(time.perf_counter() - t0)
    t = statistics.median(times)
    return {"value": round(busbw("allreduce", n * 2, t, R), 4), "unit": "GB/s", "cores": 1,
            "host_cores": host_threads(), "kind": "oracle",
            "sample": "the same IR program (%s, R=%d, bf16) on %d MiB per rank instead of the workload's size: "
                      "median of %d runs of oracle.sim.simulate (numpy, 1 thread), %.2f s per run"
                      % (algo.name, R, n * 2 // MIB, reps, t)}


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, on a bounded sample of the workload."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    R = args.ranks if args.gpus == 1 else args.gpus
    algo = build_program(args, R)
    sample = 16 * MIB
    import numpy as np
    import synth
    from oracle import irparse, sim
    al = irparse.parse(algo.to_xml())
    n = sample // 2
    xs = [synth.hashed_numpy(q, np.arange(n), "bfloat16") for q in range(R)]
    for _ in range(args.warmup):
        sim.simulate(al, xs, n, "bfloat16", "sum")
    t0 = time.perf_counter()
    for _ in range(args.steps):
        sim.simulate(al, xs, n, "bfloat16", "sum")
    t = (time.perf_counter() - t0) / args.steps
    v = busbw("allreduce", sample, t, R)
    cfg = config_dict(args, R, args.gpus)
    out = {"impl": "reference", "metric": metric_name(coll_of(args.program), args.program), "value": round(v, 4), "unit": "GB/s",
           "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 3),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
           "config": cfg,
           "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                            "host_cores": host_threads(),
                            "sample": "each step: oracle.sim.simulate of the same IR on %d MiB per rank (the "
                                      "workload is %d MiB per rank; busBW is size-independent for the oracle)"
                                      % (sample // MIB, int(args.size_mib))},
           "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def metric_name(coll="allreduce", program="ring"):
    form = {"ring": "ring", "allpairs": "all-pairs", "oneshot": "one-shot", "nvls": "multimem (NVLS)",
            "allgather": "ring", "allgather_direct": "all-pairs", "reducescatter": "ring"}.get(program, program)
    if coll == "alltoall":
        return "AllToAll busBW (GB/s), direct MSCCL-IR (two-step N=1), bf16"
    if coll in ("allgather", "reducescatter"):
        return "%s busBW (GB/s), %s MSCCL-IR, bf16" % ({"allgather": "AllGather", "reducescatter": "ReduceScatter"}[coll],
                                                      form)
    return "AllReduce busBW (GB/s), %s MSCCL-IR, bf16" % form


def config_dict(args, R, N):
    if N == 1:
        base = {"ring": "largest single-GPU analogue of BASELINE configs[1] (ring AllReduce, bf16)",
                "allpairs": "BASELINE configs[2] shape (all-pairs AllReduce)",
                "oneshot": "BASELINE configs[2] shape (one-shot AllReduce)",
                "alltoall": "BASELINE configs[3] shape (AllToAll)",
                "allgather": "BASELINE configs[4] shape (ring AllGather)",
                "allgather_direct": "BASELINE configs[4] shape (all-pairs AllGather)",
                "nvls": "BASELINE configs[1] shape with the multimem (NVLS) AllReduce program",
                "reducescatter": "BASELINE configs[4] shape (ring ReduceScatter)"}[args.program]
        mode = "%d virtual ranks on 1 B200 (HBM-bound)" % R
    else:
        base = {"ring": "BASELINE configs[1]: ring AllReduce, bf16", "allpairs": "all-pairs AllReduce",
                "oneshot": "one-shot AllReduce", "alltoall": "BASELINE configs[3]: AllToAll",
                "nvls": "multimem (NVLS) AllReduce",
                "allgather": "BASELINE configs[4]: ring AllGather",
                "allgather_direct": "BASELINE configs[4]: all-pairs AllGather", "reducescatter": "BASELINE configs[4]: ring "
                "ReduceScatter"}[args.program]
        mode = "%d B200, 1 process per GPU, CUDA IPC over NVLink" % N
    return {"workload": "%s -- MSCCL-IR %s, %d channel(s) x %d instance(s), %s protocol, %s, %d MiB per rank"
                        % (base, args.program, args.channels, args.instances, args.protocol, mode,
                           int(args.size_mib)),
            "program": args.program, "ranks": R, "bytes_per_rank": int(args.size_mib * MIB),
            "channels": args.channels, "instances": args.instances, "protocol": args.protocol,
            "split_phases": bool(args.split), "rings": args.rings,
            "threads": args.threads, "slots": args.slots, "slot_bytes": args.slot_kib * 1024,
            "l2": "inputs (%d MiB total) larger than L2 (126 MB); no flush" % int(args.size_mib * (R if N == 1 else 1)),
            "parallelism": "virtual%d" % R if N == 1 else "ranks%d" % N}


# ----------------------------------------------------------------------------- GPU helpers
def set_params(rt, args):
    rt.set_param("MSCCL_SLOTS", args.slots)
    rt.set_param("MSCCL_SLOT_BYTES", args.slot_kib * 1024)
    rt.set_param("MSCCL_THREADS", args.threads)
    rt.set_param("MSCCL_MAX_CHANNELS", max(32, args.channels * args.instances * (2 if args.split else 1)))
    rt.set_param("MSCCL_TIMEOUT_S", 60)
    rt.set_param("MSCCL_DIRECT_TILE", 2)  # every rank registers its buffers (reading R19b)


def sampled_parity(algo, recv_list, n, ranks_to_check, local=None, dtype="bfloat16"):
    """Bit-exact check of sampled outputs against the oracle's reduction trees (2-byte float
    dtypes). recv_list[i] is the output of rank (local[i] if local else i)."""
    import numpy as np
    import torch
    import synth
    from oracle import irparse, sampled
    al = irparse.parse(algo.to_xml())
    g = np.random.default_rng(1)
    idx = np.unique(np.concatenate([g.integers(0, n, SEED_SAMPLES), [0, n - 1, n // 2]]))
    bad = 0
    for i, q in enumerate(ranks_to_check):
        want = sampled.reduction_at(al, lambda r, ii: synth.hashed_numpy(r, ii, dtype), n, dtype, "sum",
                                    idx, rank=q)
        out = recv_list[q if local is None else local.index(q)]
        got = out[torch.from_numpy(idx).to(out.device)].view(torch.int16).cpu().numpy().view(np.uint16)
        bad += int(np.count_nonzero(got != np.asarray(want).view(np.uint16)))   # bit patterns
    return bad, idx.size * len(ranks_to_check)


class Ranks:
    """The ranks this process drives: all R virtual ranks (N = 1) or its one rank (N > 1).
    call(progs, sends, recvs, count) issues one collective on every local rank in one group
    (one cooperative launch per device)."""

    def __init__(self, rt, comms, ranks, R, world, dev):
        self.rt, self.comms, self.ranks, self.R, self.world, self.dev = rt, comms, ranks, R, world, dev

    def load(self, algo, lo=0, hi=0):
        return [c.load(algo.to_xml(), lo, hi) for c in self.comms]

    def unload(self, progs):
        for c, p in zip(self.comms, progs):
            c.unload(p)

    def call(self, progs, sends, recvs, count, stream=None):
        with self.rt.group():
            for c, p, s, r in zip(self.comms, progs, sends, recvs):
                c.run(p, s, r, count, stream=stream)

    def coll(self, coll, sends, recvs, stream=None):
        with self.rt.group():
            for c, s, r in zip(self.comms, sends, recvs):
                getattr(c, coll)(s, r, stream=stream)

    def tmax(self, t):
        """max over ranks of a per-rank time (device-timed), via the plumbing group."""
        if self.world == 1:
            return t
        import torch
        import torch.distributed as dist
        tt = torch.tensor([t], dtype=torch.float64)
        if dist.get_backend() == "nccl":
            tt = tt.to(self.dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        return float(tt.item())

    def per_rank(self, t):
        """every rank's own time (rank order), via the plumbing group."""
        if self.world == 1:
            return [t]
        import torch.distributed as dist
        out = [None] * self.world
        dist.all_gather_object(out, t)
        return out

    def all_ok(self, ok):
        if self.world == 1:
            return bool(ok)
        import torch
        import torch.distributed as dist
        tt = torch.tensor([1 if ok else 0], dtype=torch.int64)
        if dist.get_backend() == "nccl":
            tt = tt.to(self.dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MIN)
        return bool(tt.item())

    def barrier(self):
        if self.world > 1:
            import torch.distributed as dist
            dist.barrier()


def cur():
    """The current CUDA stream handle (the capture stream while a graph is being captured)."""
    import torch
    return torch.cuda.current_stream().cuda_stream


def timed(fn, iters, warmup, stream, graph, R, local=None):
    """Mean device time per call of fn() (CUDA events on `stream`, synchronised on both
    sides, max over ranks). fn() must issue its work on the current stream. graph=True
    captures `iters` calls into one CUDA graph and times its replay. Returns (seconds, mode)."""
    import torch
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    mode = "eager"
    run = None
    if graph:
        try:
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):   # torch's capture stream; fn() issues on the current stream
                for _ in range(iters):
                    fn()
            g.replay()
            torch.cuda.synchronize()
            run, mode = g.replay, "cuda-graph"
        except Exception as e:
            torch.cuda.synchronize()
            print("graph capture failed: %s" % e, file=sys.stderr)
            run = None
    if run is None:
        def run():
            for _ in range(iters):
                fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    R.barrier()
    torch.cuda.synchronize()
    e0.record(stream)
    run()
    e1.record(stream)
    torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / 1e3 / iters
    if local is not None:
        local[0] = t
    return R.tmax(t), mode


# ----------------------------------------------------------------------------- extras
def extras(R, stream, nccl=None, S=256 * MIB):
    """BASELINE configs[2..4] on the same ranks: 1 KiB fp16 AllReduce latency (graph replay;
    one-shot / two-shot / ring LL) and the launch floor, AllToAll at 256 MiB per rank, and
    AllGather / ReduceScatter rings at 256 MiB per rank."""
    import torch
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    W = R.R
    out = {}
    lat = {}
    n = 512  # 1 KiB of fp16 per rank
    send = [synth.hashed(q, torch.arange(n, device=R.dev), "float16") for q in R.ranks]
    recv = [torch.empty_like(x) for x in send]
    lat_regs = register_all(R, send + recv)   # N > 1: direct placement / multimem need them
    for name, algo in (("floor_nop", None), ("one_hop_LL", "hop"), ("one_hop_LL128", "hop128"),
                       ("oneshot_LL", P.oneshot_allreduce(W, protocol="LL")),
                       ("nvls_multimem", P.nvls_allreduce(W, 1)),
                       ("allpairs_LL", P.allpairs_allreduce(W, protocol="LL")),
                       ("ring_LL", P.ring_allreduce(W, protocol="LL")),
                       ("ring_ch%d_LL" % W, P.ring_allreduce(W, channels=W, protocol="LL"))):
        if algo is None:
            progs = [c.load(nop_ir(W)) for c in R.comms]
        elif algo in ("hop", "hop128"):
            progs = [c.load(hop_ir(W, "LL" if algo == "hop" else "LL128")) for c in R.comms]
        else:
            progs = R.load(algo, 0, 1 << 20)
        try:
            t, mode = timed(lambda: R.call(progs, send, recv, n), 50, 5, stream, True, R)
            lat[name] = round(t * 1e6, 2)
            lat["mode"] = mode
        except Exception as e:
            lat[name] = "error: %s" % str(e)[:160]
        R.unload(progs)
    if nccl is not None:
        t, mode = timed(lambda: nccl.allreduce(send[0], recv[0], "float16", stream=cur()), 50, 5, stream, True, R)
        lat["nccl_allreduce"] = round(t * 1e6, 2)
    lat["note"] = ("floor_nop = an MSCCL-IR program of one nop per rank: cooperative launch + prologue + "
                   "epilogue under graph replay; one_hop = rank r sends 1 KiB to rank r+1 (one message of the "
                   "protocol); the collective latencies are read against floor + hops")
    out["allreduce_1KiB_fp16_latency_us"] = lat
    for r_ in lat_regs:
        r_.deregister()
    del send, recv
    # AllToAll (direct two-step N=1), AllGather and ReduceScatter rings: S per rank (256 MiB), bf16
    n = S // 2
    nb = n // W
    specs = (("nvls_allreduce", P.nvls_allreduce(W, 32 if R.world == 1 else 8), n, n, n),
             ("nvls_reducescatter", P.nvls_reducescatter(W, 32 if R.world == 1 else 8), n, nb, nb),
             ("nvls_allgather", P.nvls_allgather(W, 32 if R.world == 1 else 8), nb, n, nb),
             ("alltoall", P.alltoall_twostep(1, W, instances=2 if R.world == 1 else 4), n, n, nb),
             ("allgather", P.ring_allgather(W, 1, 32 if R.world == 1 else 8), nb, n, nb),
             ("reducescatter", P.ring_reducescatter(W, 1, 32 if R.world == 1 else 8), n, nb, nb))
    for coll, algo, ins, outs, cnt in specs:
        progs = R.load(algo)
        send = [synth.hashed(q, torch.arange(ins, device=R.dev), "bfloat16") for q in R.ranks]
        recv = [torch.empty(outs, dtype=torch.bfloat16, device=R.dev) for _ in R.ranks]
        regs = register_all(R, send + recv)
        t, mode = timed(lambda: R.call(progs, send, recv, cnt), 5, 2, stream, False, R)
        if coll == "alltoall":
            ok = check_alltoall(R, recv, W, n)
        elif coll in ("allgather", "nvls_allgather"):
            ok = check_allgather(R, recv, W, nb)
        elif coll == "nvls_allreduce":
            ranks = [q for q in (0, W - 1) if q in R.ranks]
            bad, _ = sampled_parity(algo, recv, n, ranks, local=R.ranks)
            ok = bad == 0
        else:
            ranks = [q for q in (0, W - 1) if q in R.ranks]
            bad, _ = sampled_parity(algo, recv, nb, ranks, local=R.ranks)
            ok = bad == 0
        base_coll = coll.replace("nvls_", "")
        ent = {"busbw_GBps": round(busbw(base_coll, S, t, W), 2),
               "ms": round(t * 1e3, 3),
               "ctas_per_rank": int(progs[0].info()["thread_blocks"]), "bit_exact": R.all_ok(ok)}
        if nccl is not None and not coll.startswith("nvls_"):
            fn = {"alltoall": lambda: nccl.alltoall(send[0], recv[0], "bfloat16", W, cur()),
                  "allgather": lambda: nccl.allgather(send[0], recv[0], "bfloat16", cur()),
                  "reducescatter": lambda: nccl.reducescatter(send[0], recv[0], "bfloat16", "sum", cur())}[coll]
            tn, _ = timed(fn, 5, 2, stream, False, R)
            ent["nccl_busbw_GBps"] = round(busbw(coll, S, tn, W), 2)
        out["%s_bf16_%dMiB" % (coll, S // MIB)] = ent
        for r_ in regs:
            r_.deregister()
        R.unload(progs)
        del send, recv
        torch.cuda.empty_cache()
    return out


def check_alltoall(R, recv, W, n):
    import torch
    import synth
    ok = True
    for i, q in enumerate(R.ranks):
        if q not in (0, W - 1):
            continue
        for p in range(W):
            src = synth.hashed(p, torch.arange(q * (n // W), (q + 1) * (n // W), device=R.dev), "bfloat16")
            ok = ok and torch.equal(recv[i].view(W, -1)[p], src)
    return ok


def check_allgather(R, recv, W, nb):
    import torch
    import synth
    ok = True
    for i, q in enumerate(R.ranks):
        if q not in (0, W - 1):
            continue
        for p in range(W):
            ok = ok and torch.equal(recv[i].view(W, -1)[p], synth.hashed(p, torch.arange(nb, device=R.dev),
                                                                         "bfloat16"))
    return ok


def register_all(R, tensors):
    """N > 1: register the user buffers for direct placement (reading R15b), collectively."""
    if R.world == 1 or getattr(R, "no_register", False):
        return []
    from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
    return [mdist.register(R.comms[0], t) for t in tensors]


# ----------------------------------------------------------------------------- sweep
def sweep(R, stream, path, max_mib, nccl=None):
    """Per-size JSON lines: AllReduce (the size-range program set of
    programs.tuned_allreduce) and AllToAll (programs.tuned_alltoall), 1 KiB .. max per rank,
    eager and CUDA graph; 20 warm-up + 50 timed ops, and 1000 for the <= 64 KiB
    latency mode. Correctness of the last op: bit-exact sampled parity (AllReduce, oracle
    reduction trees) / exact permutation (AllToAll)."""
    import torch
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    W = R.R
    f = open(path, "w") if path else None
    impl_sets = {"allreduce": P.tuned_allreduce(W), "allreduce_multimem": P.tuned_allreduce_multimem(W),
                 "alltoall": P.tuned_alltoall(W)}
    lines = []
    for label in ("allreduce", "allreduce_multimem", "alltoall"):
        coll = "allreduce" if label.startswith("allreduce") else label
        if label == "allreduce_multimem" and nccl is not None:
            pass  # NCCL runs once per collective, with the first AllReduce set
        sets = [(algo, lo, hi, R.load(algo, lo, hi)) for algo, lo, hi in impl_sets[label]]
        size = 1024
        while size <= max_mib * MIB:
            n = size // 2
            send = [synth.hashed(q, torch.arange(n, device=R.dev), "bfloat16") for q in R.ranks]
            recv = [torch.empty_like(x) for x in send]
            regs = register_all(R, send + recv)
            per = (n // W) * 2 if coll == "alltoall" else size   # selection bytes (count * w)
            chosen = next(a for a, lo, hi, _ in sets if lo <= per and (hi == 0 or per < hi))
            impls = [("msccl", lambda: R.coll(coll, send, recv))]
            if nccl is not None and label != "allreduce_multimem":
                impls.append(("nccl", (lambda: nccl.allreduce(send[0], recv[0], "bfloat16", stream=cur()))
                              if coll == "allreduce" else
                              (lambda: nccl.alltoall(send[0], recv[0], "bfloat16", W, cur()))))
            for impl, fn in impls:
                for graph in (False, True):
                    iters = 50 if size <= 256 * MIB else 20
                    t_local = [0.0]
                    t, mode = timed(fn, iters, 20, stream, graph, R, t_local)
                    rec = {"impl": impl, "coll": coll, "set": label, "program": chosen.name if impl == "msccl" else "nccl",
                           "R": W, "dtype": "bf16", "op": "sum", "bytes": size, "count": n,
                           "iters": iters, "warmup": 20, "graph": mode == "cuda-graph", "t_us_max": round(t * 1e6, 3),
                           "t_us_per_rank": [round(x * 1e6, 3) for x in R.per_rank(t_local[0])],
                           "algbw": round(size / t / 1e9, 3), "busbw": round(busbw(coll, size, t, W), 3)}
                    if impl == "msccl":
                        rec.update({"proto": chosen.proto, "instances": chosen.ninstances,
                                    "channels": chosen.nchannels, "ctas_per_rank": chosen.max_tbs(),
                                    "slots": R.rt.get_param("MSCCL_SLOTS"),
                                    "slot_bytes": R.rt.get_param({"LL": "MSCCL_LL_SLOT_BYTES",
                                                                  "LL128": "MSCCL_LL128_SLOT_BYTES"}.get(
                                                                      chosen.proto, "MSCCL_SLOT_BYTES"))})
                    if R.world > 1:
                        rec["frac_nvlink"] = round(rec["busbw"] / NVLINK_NOMINAL, 4)
                    if size <= 64 * 1024 and graph:
                        tl, _ = timed(fn, 1000, 20, stream, True, R)
                        rec["latency_mode_us"] = round(tl * 1e6, 3)
                    if impl == "msccl":
                        if coll == "allreduce":
                            ranks = [q for q in (0, W - 1) if q in R.ranks]
                            bad, _ = sampled_parity(chosen, recv, n, ranks, local=R.ranks)
                            rec["correct"] = R.all_ok(bad == 0)
                        else:
                            rec["correct"] = R.all_ok(check_alltoall(R, recv, W, n))
                    lines.append(rec)
                    if int(os.environ.get("RANK", "0")) == 0:
                        print(json.dumps(rec), flush=True)
                        if f:
                            f.write(json.dumps(rec) + "\n")
                            f.flush()
            for r_ in regs:
                r_.deregister()
            del send, recv
            torch.cuda.empty_cache()
            size *= 2
        for _, _, _, progs in sets:
            R.unload(progs)
    if f:
        f.close()
    return lines


# ----------------------------------------------------------------------------- N = 1
def run_virtual(args):
    import torch
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
    W = args.ranks
    set_params(rt, args)
    algo = build_program(args, W)
    ir_text = algo.to_xml()
    S = int(args.size_mib * MIB)
    n = S // 2
    dev = torch.device("cuda:0")
    comms = rt.Comm.virtual(W, 0)
    R = Ranks(rt, comms, list(range(W)), W, 1, dev)
    stream = torch.cuda.current_stream()
    if args.sweep:
        rt.set_param("MSCCL_MAX_CHANNELS", 64)
        sweep(R, stream, args.sweep, args.sweep_max_mib)
        return None
    progs = [c.load(ir_text) for c in comms]
    direct = rt.get_param("MSCCL_DIRECT") != 0 and args.protocol == "Simple"
    touches = [p.touches(direct) for p in progs]
    coll = coll_of(args.program)
    ns, nr, count = shapes(coll, n, W)
    idx = torch.arange(ns, device=dev, dtype=torch.int64)
    send = [synth.hashed(q, idx, "bfloat16") for q in range(W)]
    del idx
    recv = [torch.empty(nr, dtype=torch.bfloat16, device=dev) for _ in range(W)]

    def step():
        R.call(progs, send, recv, count, stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    clocks = Clocks(0)
    clocks.start()
    time.sleep(0.3)
    l0 = rt.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    ev0.record(stream)
    for _ in range(args.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize()
    t = ev0.elapsed_time(ev1) / 1e3 / args.steps
    launches = rt.launch_count() - l0
    clk = clocks.stop()
    for c in comms:
        if c.async_error():
            raise RuntimeError("watchdog fired during the bench")
    if coll == "alltoall":
        ok = check_alltoall(R, recv, W, n)
        bad, total = (0 if ok else 1), 2 * n
    elif coll == "allgather":
        ok = check_allgather(R, recv, W, count)
        bad, total = (0 if ok else 1), 2 * n
    else:
        bad, total = sampled_parity(algo, recv, count, [0, W - 1])
    res = {"t": t, "coll": coll, "launches": launches, "clocks": clk, "parity_bad": bad, "parity_total": total,
           "algo": algo, "S": S, "R": W, "touches": touches, "direct": direct}
    if not args.no_e2e:
        res["e2e"] = e2e(R, send, recv, lambda sn, rc, st: R.call(progs, sn, rc, count, st), S, coll, W,
                         args.steps, stream)
    R.unload(progs)
    if not args.quiet_extra:
        del send, recv
        torch.cuda.empty_cache()
        res["extras"] = extras(R, stream)
    for c in comms:
        c.destroy()
    return res


def e2e(R, send, recv, call, S, coll, W, steps, stream):
    """The same metric end to end through the public API: every step copies that step's
    inputs from pinned host memory to the device, runs the collective, and reads the result
    back (every local rank); max over ranks.

    Steps are software-pipelined over two device buffer sets and three streams: the H2D of
    step k+1 and the D2H of step k-1 overlap the collective of step k. Every step still pays
    its own copies inside the timed region; only independent work overlaps. PCIe moves data
    in both directions at once. `serial_ms` is the same loop with each step's three phases
    run back to back on one stream."""
    import torch
    host_in = [s_.cpu().pin_memory() for s_ in send]
    sets = [(send, recv), ([torch.empty_like(x) for x in send], [torch.empty_like(x) for x in recv])]
    host_out = [[torch.empty(r.numel(), dtype=r.dtype).pin_memory() for r in recv] for _ in range(2)]
    k = max(4, min(32, steps))   # the bench's K steps (pipeline fill / drain amortised like the device-timed loop)
    s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
    ev = lambda: torch.cuda.Event()
    h2d_done = [ev(), ev()]
    coll_done = [ev(), ev()]
    d2h_done = [ev(), ev()]

    def pipelined_step(i):
        b = i % 2
        snd, rcv = sets[b]
        with torch.cuda.stream(s_in):
            s_in.wait_event(coll_done[b])        # step i-2 has finished reading snd
            for d, h in zip(snd, host_in):
                d.copy_(h, non_blocking=True)
            h2d_done[b].record(s_in)
        stream.wait_event(h2d_done[b])
        stream.wait_event(d2h_done[b])           # step i-2's result has left rcv
        call(snd, rcv, stream)
        coll_done[b].record(stream)
        with torch.cuda.stream(s_out):
            s_out.wait_event(coll_done[b])
            for r, h in zip(rcv, host_out[b]):
                h.copy_(r, non_blocking=True)
            d2h_done[b].record(s_out)

    def serial_step():
        for d, h in zip(send, host_in):
            d.copy_(h, non_blocking=True)
        call(send, recv, stream)
        for r, h in zip(recv, host_out[0]):
            h.copy_(r, non_blocking=True)

    for i in range(2):
        pipelined_step(i)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    R.barrier()
    torch.cuda.synchronize()
    e0.record(stream)
    for i in range(k):
        pipelined_step(i)
    stream.wait_stream(s_out)
    e1.record(stream)
    torch.cuda.synchronize()
    te = R.tmax(e0.elapsed_time(e1) / 1e3 / k)
    serial_step()
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(2):
        serial_step()
    e1.record(stream)
    torch.cuda.synchronize()
    ts = R.tmax(e0.elapsed_time(e1) / 1e3 / 2)
    h2d = sum(x.numel() * x.element_size() for x in send)
    d2h = sum(x.numel() * x.element_size() for x in recv)
    return {"value": round(busbw(coll, S, te, W), 3), "unit": "GB/s",
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "ms_per_step": round(te * 1e3, 3),
            "serial_ms_per_step": round(ts * 1e3, 3),
            "note": "C-ABI call with pinned host buffers: H2D of this process's %d rank input(s) + collective + "
                    "D2H of the output(s) every step, pipelined over 2 buffer sets (PCIe-bound)" % len(send)}


# ----------------------------------------------------------------------------- N > 1
def peer_copy_peak(rank, world, dev):
    """Measured one-direction peer copy GB/s between this GPU and the next (1 GiB, best of
    5, CUDA events), the NVLink roofline denominator; None when GPUs are shared."""
    import torch
    if os.environ.get("MSCCL_FORCE_DEVICE") or torch.cuda.device_count() < 2:
        return None
    peer = (dev.index + 1) % torch.cuda.device_count()
    a = torch.empty(1 << 30, dtype=torch.uint8, device=dev)
    b = torch.empty(1 << 30, dtype=torch.uint8, device=torch.device("cuda", peer))
    best = 0.0
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        b.copy_(a, non_blocking=True)
        e1.record()
        torch.cuda.synchronize()
        best = max(best, (1 << 30) / (e0.elapsed_time(e1) / 1e3) / 1e9)
    del a, b
    torch.cuda.empty_cache()
    return round(best, 1)


def run_multi(args, rank, world, local_rank):
    import torch
    forced = os.environ.get("MSCCL_FORCE_DEVICE")
    if forced:  # testing the multi-process path on one GPU only
        local_rank = int(forced)
    import torch.distributed as dist
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if forced:  # NCCL refuses two ranks on one GPU; plumbing only anyway
        dist.init_process_group("gloo", rank=rank, world_size=world)
    else:
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
    set_params(rt, args)
    from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
    comm = mdist.init_from_process_group(local_rank)
    R = Ranks(rt, [comm], [rank], world, world, dev)
    R.no_register = args.no_register
    stream = torch.cuda.current_stream()
    nccl, nccl_note = None, None
    if args.no_nccl:
        nccl_note = "skipped (--no-nccl)"
    elif forced:
        nccl_note = "skipped: every rank is on one GPU (MSCCL_FORCE_DEVICE); NCCL refuses duplicate GPUs"
    else:
        try:
            sys.path.insert(0, os.path.join(ROOT, "tools"))
            import nccl_arm
            nccl = nccl_arm.Nccl().init(rank, world)
            nccl_note = "NCCL %d via ctypes (torch-bundled libnccl.so.2), default env" % nccl.version
        except Exception as e:
            nccl, nccl_note = None, "unavailable: %s" % str(e)[:200]
    if args.sweep:
        rt.set_param("MSCCL_MAX_CHANNELS", 64)
        sweep(R, stream, args.sweep if rank == 0 else None, args.sweep_max_mib, nccl)
        if nccl:
            nccl.destroy()
        comm.destroy()
        dist.destroy_process_group()
        return None
    peak_peer = peer_copy_peak(rank, world, dev)
    algo = build_program(args, world)
    progs = R.load(algo)
    S = int(args.size_mib * MIB)
    n = S // 2
    coll = coll_of(args.program)
    ns, nr, count = shapes(coll, n, world)
    send = [synth.hashed(rank, torch.arange(ns, device=dev, dtype=torch.int64), "bfloat16")]
    recv = [torch.empty(nr, dtype=torch.bfloat16, device=dev)]
    regs = register_all(R, send + recv)
    h0 = comm.stats()["cross_direct_handshakes"]

    def step():
        R.call(progs, send, recv, count, stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    clocks = Clocks(local_rank) if rank == 0 else None
    if clocks:
        clocks.start()
        time.sleep(0.3)
    l0 = rt.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    dist.barrier()
    ev0.record(stream)
    for _ in range(args.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize()
    dist.barrier()
    t = R.tmax(ev0.elapsed_time(ev1) / 1e3 / args.steps)
    launches = rt.launch_count() - l0
    clk = clocks.stop() if clocks else None
    handshakes = comm.stats()["cross_direct_handshakes"] - h0
    if coll == "alltoall":
        ok = check_alltoall(R, recv, world, n)
        bad, total = (0 if ok else 1), n
    elif coll == "allgather":
        ok = check_allgather(R, recv, world, count)
        bad, total = (0 if ok else 1), n
    else:
        bad, total = sampled_parity(algo, recv, count, [rank], local=[rank])
    bt = torch.tensor([bad, total, handshakes], dtype=torch.int64)
    if dist.get_backend() == "nccl":
        bt = bt.to(dev)
    dist.all_reduce(bt)
    bad, total, handshakes = (int(x) for x in bt.tolist())
    res = {"t": t, "coll": coll, "launches": launches, "clocks": clk, "parity_bad": bad, "parity_total": total,
           "algo": algo, "S": S, "R": world, "peak_peer": peak_peer, "nccl_note": nccl_note,
           "direct_handshakes": handshakes, "registered": not args.no_register}
    if nccl is not None:
        fn = {"allreduce": lambda: nccl.allreduce(send[0], recv[0], "bfloat16", stream=cur()),
              "alltoall": lambda: nccl.alltoall(send[0], recv[0], "bfloat16", world, cur()),
              "allgather": lambda: nccl.allgather(send[0], recv[0], "bfloat16", cur()),
              "reducescatter": lambda: nccl.reducescatter(send[0], recv[0], "bfloat16", "sum", cur())}[coll]
        tn, _ = timed(fn, args.steps, args.warmup, stream, False, R)
        res["nccl"] = {"value": round(busbw(coll, S, tn, world), 3), "ms_per_step": round(tn * 1e3, 4),
                       "note": nccl_note}
    if not args.no_e2e:
        res["e2e"] = e2e(R, send, recv, lambda sn, rc, st: R.call(progs, sn, rc, count, st), S, coll, world,
                         args.steps, stream)
    for r_ in regs:
        r_.deregister()
    R.unload(progs)
    del send, recv
    torch.cuda.empty_cache()
    if not args.quiet_extra:
        res["extras"] = extras(R, stream, nccl, S)
    if rank == 0 and not args.no_cpu:
        res["cpu_baseline"] = cpu_oracle_run(world, algo, 32 * MIB)
    if nccl:
        nccl.destroy()
    comm.destroy()
    dist.destroy_process_group()
    return res if rank == 0 else None


# ----------------------------------------------------------------------------- main
def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    N = world if world > 1 else args.gpus
    if world > 1:
        res = run_multi(args, rank, world, local_rank)
        if rank != 0 or res is None:
            return
    else:
        res = run_virtual(args)
        if res is None:
            return
    R = res["R"]
    S, t, algo = res["S"], res["t"], res["algo"]
    coll = res.get("coll", "allreduce")
    value = busbw(coll, S, t, R)
    launches_per_step = max(1, res["launches"] // args.steps)
    out = {
        "metric": metric_name(coll, args.program), "value": round(value, 3), "unit": "GB/s", "n_gpus": N,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 4),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
        "data": "synthetic (counter-based uniform[-1,1) bf16, seed 20230325+rank)",
        "config": config_dict(args, R, N),
    }
    if world > 1:
        # one rank per GPU: the bytes cross NVLink. Egress per rank per step = busBW * t, so
        # busBW is the achieved per-direction link bandwidth.
        pk = res.get("peak_peer")
        peak, src = (pk, "measured peer copy (1 GiB cudaMemcpyPeer, this box)") if pk else \
            (770.0, "fallback: B200_PROFILING.md measured peer copy per direction (no 2nd GPU to measure)")
        out["roofline"] = {"bound": "nvlink", "achieved": round(value, 1), "peak": peak, "unit": "GB/s",
                           "frac": round(value / peak, 4), "traffic": None, "peak_source": src,
                           "frac_nominal_900": round(value / NVLINK_NOMINAL, 4),
                           "kernel": "mscclInterpreter<bf16,%s,Simple>" % ("copy" if coll == "alltoall" else "sum"),
                           "algorithmic_bytes_per_launch": int(S * (2 if coll == "allreduce" else 1) * (R - 1) / R),
                           "launch_ms": round(t * 1e3 / launches_per_step, 4)}
        out["frac_nvlink"] = round(value / NVLINK_NOMINAL, 4)
        out["direct_placement"] = {"registered_buffers": res["registered"],
                                   "cross_launch_handshakes": res["direct_handshakes"]}
        out["nccl"] = res.get("nccl", {"note": res.get("nccl_note")})
    else:
        # All R virtual ranks run in one launch on one GPU: the HBM bytes any implementation
        # must move are every rank's input read once and its output written once.
        peak, peak_src = measured_peak()
        ns, nr, _ = shapes(coll, S // 2, R)
        per_chunk = ns * 2 / algo.gpus[0].i_chunks       # E * w: every buffer's chunk size
        alg_bytes = sum(res["touches"]) * per_chunk
        launch_s = t / launches_per_step
        compulsory = (ns + nr) * 2 * R                     # inputs read once + outputs written once
        hbm_achieved = compulsory / launch_s / 1e9
        achieved = alg_bytes / launch_s / 1e9
        traffic, prof = ncu_traffic()
        l2peak, l2src = l2_peak()
        is_default = (args.program, args.instances, args.channels, args.slot_kib, args.threads, args.protocol,
                      args.split, args.rings) == ("ring", 32, 1, 256, 256, "Simple", False, 1)
        out["roofline"] = {
            "bound": "hbm", "achieved": round(hbm_achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(hbm_achieved / peak, 4), "traffic": traffic if is_default else None,
            "peak_source": peak_src,
            "kernel": "mscclInterpreter<bf16,%s,Simple>" % ("copy" if coll == "alltoall" else "sum"),
            "algorithmic_bytes_per_launch": int(compulsory), "launch_ms": round(launch_s * 1e3, 4),
            "note": "algorithmic = compulsory HBM bytes of one launch covering all %d ranks: every input read "
                    "once + every output written once (2 S R for AllReduce); traffic = ncu dram read+write bytes per launch "
                    "(profiles/ncu_summary.json, default config only)" % R,
            "l2": {"touched_bytes_per_launch": int(alg_bytes), "achieved": round(achieved, 1),
                   "peak": l2peak, "frac": round(achieved / l2peak, 4) if l2peak else None,
                   "peak_source": l2src,
                   "note": "touched = the program's per-instruction operand bytes (send 2, recv 2, copy 2, "
                           "reduce/rrc/rrs 3, rrcs 4, rcs 3 chunks; a direct recv 0, a direct rcs 2, a pulled send 0), i.e. "
                           "the L2-level traffic of the interpreter; FIFO slots live mostly in L2"},
            "direct_placement": res.get("direct")}
        out["nccl"] = {"note": "skipped: one GPU (NCCL cannot run 8 ranks on one device); the NCCL arm runs "
                               "under torchrun with N > 1"}
    out["gpu_launches"] = res["launches"]
    out["parity"] = {"sampled_outputs": res["parity_total"], "mismatches": res["parity_bad"],
                     "against": "oracle reduction trees (oracle/sampled.py), bit-exact"}
    out["clocks"] = res["clocks"]
    if "e2e" in res:
        out["e2e"] = res["e2e"]
    if "extras" in res:
        out["extras"] = res["extras"]
    if world == 1 and not args.no_cpu:
        out["cpu_baseline"] = cpu_oracle_run(R, algo, 32 * MIB)
    elif "cpu_baseline" in res:
        out["cpu_baseline"] = res["cpu_baseline"]
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
