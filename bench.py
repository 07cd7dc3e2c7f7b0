#!/usr/bin/env python3
"""Benchmark of the MSCCL-IR interpreter (MSCCLang, ASPLOS '23) on B200.

Metric (BASELINE.json): AllReduce / AllToAll bus bandwidth (nccl-tests convention,
busBW = S/t * 2(R-1)/R for AllReduce, S = bytes per rank) — one JSON line on stdout.

Workload of the default run (N=1, one GPU): BASELINE config 1 — ring AllReduce, bf16,
8 channels, pipelined chunks — executed by R=8 VIRTUAL ranks on one B200 (all ranks'
buffers and FIFOs in that GPU's HBM, one cooperative interpreter launch per step), at
S = 256 MiB per rank (inputs 2 GiB > 126 MB L2, so no L2 flush is needed). With one GPU
the "links" are HBM: the roofline is HBM bandwidth.

Under torchrun (N>1) each process drives one GPU as one rank over CUDA IPC peer memory
(NVLink/NVSwitch): ring AllReduce over N ranks, S per rank fixed ("weak"), value = busBW
from the max over ranks of the CUDA-event time.

`--impl reference` times the CPU oracle (oracle/sim.py) executing the same program on a
bounded sample of the same workload, on the host cores.
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


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="msccl", choices=["msccl", "reference"])
    ap.add_argument("--ranks", type=int, default=8, help="virtual ranks when N=1")
    ap.add_argument("--size-mib", type=float, default=256.0, help="bytes per rank (MiB)")
    ap.add_argument("--program", default="ring", choices=["ring", "allpairs", "oneshot", "alltoall"])
    ap.add_argument("--channels", type=int, default=1)
    ap.add_argument("--instances", type=int, default=32)
    ap.add_argument("--protocol", default="Simple")
    ap.add_argument("--threads", type=int, default=256)
    ap.add_argument("--slots", type=int, default=4)
    ap.add_argument("--slot-kib", type=int, default=256)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--quiet-extra", action="store_true", help="skip the small-message and AllToAll extras")
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
        return P.ring_allreduce(R, channels=args.channels, instances=args.instances, protocol=args.protocol)
    if args.program == "allpairs":
        return P.allpairs_allreduce(R, instances=args.instances, protocol=args.protocol)
    if args.program == "oneshot":
        return P.oneshot_allreduce(R, instances=args.instances, protocol=args.protocol)
    return P.alltoall_twostep(1, R, instances=args.instances, protocol=args.protocol)


def simple_bytes_per_rank(algo, rank, S_per_chunk):
    """Algorithmic HBM bytes of one launch for one rank under the FIFO protocol: each
    instruction reads/writes its operands once per chunk."""
    touches = {"s": 2, "r": 2, "cpy": 2, "re": 3, "rrc": 3, "rrs": 3, "rrcs": 4, "rcs": 3, "nop": 0}
    g = algo.gpus[rank]
    return sum(touches[st.op] * st.cnt for tb in g.tbs for st in tb.steps) * S_per_chunk


# ----------------------------------------------------------------------------- CPU oracle
def cpu_oracle_run(args, R, algo, sample_bytes, reps=3):
    """Time oracle.sim.simulate on a bounded sample (same program, same dtype)."""
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
            "host_cores": len(os.sched_getaffinity(0)), "kind": "oracle",
            "sample": "ring AllReduce R=%d bf16, %d MiB per rank (median of %d runs of oracle.sim.simulate, "
                      "numpy, 1 thread), %.2f s per run" % (R, n * 2 // MIB, reps, t)}


def run_reference(args):
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
    out = {"impl": "reference", "metric": metric_name(), "value": round(v, 4), "unit": "GB/s",
           "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 3),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
           "config": cfg,
           "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                            "host_cores": len(os.sched_getaffinity(0)),
                            "sample": "oracle.sim.simulate of the same IR, %d MiB per rank per step" % (sample // MIB)},
           "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def metric_name(coll="allreduce"):
    if coll == "alltoall":
        return "AllToAll busBW (GB/s), direct MSCCL-IR (two-step N=1), bf16"
    return "AllReduce busBW (GB/s), ring MSCCL-IR, bf16"


def config_dict(args, R, N):
    mode = "virtual ranks on 1 GPU" if N == 1 else "1 process per GPU, CUDA IPC peer memory"
    what = {"ring": "BASELINE config 1: ring AllReduce", "allpairs": "BASELINE config 2: all-pairs AllReduce",
            "oneshot": "BASELINE config 2: one-shot AllReduce",
            "alltoall": "BASELINE config 3: direct AllToAll"}[args.program]
    return {"workload": "%s MSCCL-IR, %d channels, %d instances, %s protocol, %d ranks (%s), %d MiB per rank"
                        % (what, args.channels, args.instances, args.protocol, R, mode, int(args.size_mib)),
            "program": args.program, "ranks": R, "bytes_per_rank": int(args.size_mib * MIB),
            "channels": args.channels, "instances": args.instances, "protocol": args.protocol,
            "threads": args.threads, "slots": args.slots, "slot_bytes": args.slot_kib * 1024,
            "l2": "inputs (%d MiB total) larger than L2 (126 MB); no flush" % int(args.size_mib * R),
            "parallelism": "virtual%d" % R if N == 1 else "ranks%d" % N}


# ----------------------------------------------------------------------------- GPU runs
def set_params(rt, args):
    rt.set_param("MSCCL_SLOTS", args.slots)
    rt.set_param("MSCCL_SLOT_BYTES", args.slot_kib * 1024)
    rt.set_param("MSCCL_THREADS", args.threads)
    rt.set_param("MSCCL_MAX_CHANNELS", max(32, args.channels * args.instances))
    rt.set_param("MSCCL_TIMEOUT_S", 30)


def sampled_parity(algo, recv_list, n, ranks_to_check):
    """Bit-exact check of sampled outputs against the oracle's reduction trees."""
    import numpy as np
    import torch
    import synth
    from oracle import irparse, sampled
    al = irparse.parse(algo.to_xml())
    g = np.random.default_rng(1)
    idx = np.unique(np.concatenate([g.integers(0, n, SEED_SAMPLES), [0, n - 1, n // 2]]))
    bad = 0
    for q in ranks_to_check:
        want = sampled.reduction_at(al, lambda r, i: synth.hashed_numpy(r, i, "bfloat16"), n, "bfloat16", "sum",
                                      idx, rank=q)
        got = recv_list[q][torch.from_numpy(idx).to(recv_list[q].device)].view(torch.int16).cpu().numpy() \
            .view(np.uint16)
        bad += int(np.count_nonzero(got != want))
    return bad, idx.size * len(ranks_to_check)


def run_virtual(args):
    import torch
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
    R = args.ranks
    set_params(rt, args)
    algo = build_program(args, R)
    ir_text = algo.to_xml()
    S = int(args.size_mib * MIB)
    n = S // 2
    dev = torch.device("cuda:0")
    comms = rt.Comm.virtual(R, 0)
    progs = [c.load(ir_text) for c in comms]
    direct = rt.get_param("MSCCL_DIRECT") != 0 and args.protocol == "Simple"
    touches = [p.touches(direct) for p in progs]
    idx = torch.arange(n, device=dev, dtype=torch.int64)
    send = [synth.hashed(q, idx, "bfloat16") for q in range(R)]
    del idx
    recv = [torch.empty(n, dtype=torch.bfloat16, device=dev) for _ in range(R)]
    stream = torch.cuda.current_stream()

    coll = "alltoall" if args.program == "alltoall" else "allreduce"

    def step():
        with rt.group():
            for q in range(R):
                if coll == "alltoall":
                    comms[q].alltoall(send[q], recv[q], stream=stream)
                else:
                    comms[q].allreduce(send[q], recv[q], stream=stream)

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
    if coll == "alltoall":  # bit-exact block permutation on the first and last rank
        bad = sum(int(torch.count_nonzero(recv[q].view(R, -1)[p] != send[p].view(R, -1)[q]))
                  for q in (0, R - 1) for p in range(R))
        total = 2 * n
    else:
        bad, total = sampled_parity(algo, recv, n, [0, R - 1])
    res = {"t": t, "coll": coll, "launches": launches, "clocks": clk, "parity_bad": bad, "parity_total": total,
           "algo": algo, "S": S, "R": R, "touches": touches, "direct": direct}
    # end-to-end through the public API with host buffers (pinned), every step
    if not args.no_e2e:
        host_in = [s.cpu().pin_memory() for s in send]
        host_out = [torch.empty(n, dtype=torch.bfloat16).pin_memory() for _ in range(R)]
        e2e_steps = max(2, min(5, args.steps))

        def e2e_step():
            for q in range(R):
                send[q].copy_(host_in[q], non_blocking=True)
            step()
            for q in range(R):
                host_out[q].copy_(recv[q], non_blocking=True)

        e2e_step()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(e2e_steps):
            e2e_step()
        e1.record(stream)
        torch.cuda.synchronize()
        te = e0.elapsed_time(e1) / 1e3 / e2e_steps
        res["e2e"] = {"value": round(busbw("allreduce", S, te, R), 3), "unit": "GB/s",
                      "h2d_bytes_per_step": S * R, "d2h_bytes_per_step": S * R,
                      "ms_per_step": round(te * 1e3, 3),
                      "note": "C-ABI call with pinned host buffers: H2D of all %d ranks' inputs + AllReduce + "
                              "D2H of all outputs per step (PCIe-bound)" % R}
    if not args.quiet_extra:
        del send, recv
        torch.cuda.empty_cache()
        res["extras"] = virtual_extras(comms, R, stream)
    for c in comms:
        c.destroy()
    return res


def _timed(fn, iters, stream, graph=True):
    """Mean device time per call of fn(); CUDA-graph replay of `iters` calls when possible."""
    import torch
    fn()
    torch.cuda.synchronize()
    mode = "eager"
    if graph:
        try:
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(iters):
                    fn()
            g.replay()
            torch.cuda.synchronize()
            run = g.replay
            mode = "cuda-graph"
        except Exception as e:
            torch.cuda.synchronize()
            print("graph capture failed: %s" % e, file=sys.stderr)
            run = None
    if mode == "eager":
        def run():
            for _ in range(iters):
                fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    run()
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(5):
        run()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / 1e3 / (5 * iters), mode


def virtual_extras(comms, R, stream):
    """BASELINE configs 3 and 4 on the same virtual ranks: 1 KB AllReduce latency (LL
    one-shot / two-shot / ring) and AllToAll busBW at 256 MiB per rank."""
    import torch
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
    dev = torch.device("cuda:0")
    out = {}
    lat = {}
    n = 512  # 1 KiB of fp16 per rank
    send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(R)]
    recv = [torch.empty_like(x) for x in send]
    for name, algo in (("oneshot_LL", P.oneshot_allreduce(R, protocol="LL")),
                       ("allpairs_LL", P.allpairs_allreduce(R, protocol="LL")),
                       ("ring_LL", P.ring_allreduce(R, protocol="LL"))):
        progs = [c.load(algo.to_xml()) for c in comms]

        def call():
            with rt.group():
                for q in range(R):
                    comms[q].run(progs[q], send[q], recv[q], n)  # current stream (graph capture)
        try:
            t, mode = _timed(call, 50, stream)
            lat[name] = round(t * 1e6, 2)
            lat["mode"] = mode
        except Exception as e:
            lat[name] = "error: %s" % str(e)[:120]
        for c, p in zip(comms, progs):
            c.unload(p)
    out["allreduce_1KiB_fp16_latency_us"] = lat
    # AllToAll (direct, N=1 two-step), 256 MiB per rank, bf16
    S = 256 * MIB
    n = S // 2
    algo = P.alltoall_twostep(1, R, instances=2)
    progs = [c.load(algo.to_xml()) for c in comms]
    send = [synth.hashed(q, torch.arange(n, device=dev), "bfloat16") for q in range(R)]
    recv = [torch.empty_like(x) for x in send]

    def a2a():
        with rt.group():
            for q in range(R):
                comms[q].run(progs[q], send[q], recv[q], n // R, stream=stream)
    t, mode = _timed(a2a, 3, stream, graph=False)
    ok = all(torch.equal(recv[q].view(R, -1)[p], send[p].view(R, -1)[q]) for q in (0, R - 1) for p in range(R))
    out["alltoall_bf16_256MiB"] = {"busbw_GBps": round(busbw("alltoall", S, t, R), 2), "ms": round(t * 1e3, 3),
                                   "ctas": sum(p.info()["thread_blocks"] for p in progs), "bit_exact": bool(ok)}
    for c, p in zip(comms, progs):
        c.unload(p)
    del send, recv
    # AllGather / ReduceScatter rings (config 5), S = 256 MiB of output (AG) / input (RS) per rank
    nb = n // R
    for name, algo, coll in (("allgather", P.ring_allgather(R, 1, 32), "allgather"),
                             ("reducescatter", P.ring_reducescatter(R, 1, 32), "reducescatter")):
        progs = [c.load(algo.to_xml()) for c in comms]
        ins = nb if coll == "allgather" else n
        outs = n if coll == "allgather" else nb
        send = [synth.hashed(q, torch.arange(ins, device=dev), "bfloat16") for q in range(R)]
        recv = [torch.empty(outs, dtype=torch.bfloat16, device=dev) for _ in range(R)]

        def call():
            with rt.group():
                for q in range(R):
                    comms[q].run(progs[q], send[q], recv[q], nb)
        t, mode = _timed(call, 3, stream, graph=False)
        if coll == "allgather":
            ok = all(torch.equal(recv[q].view(R, -1)[p], send[p]) for q in (0, R - 1) for p in range(R))
        else:
            bad, _ = sampled_parity(algo, recv, nb, [0, R - 1])
            ok = bad == 0
        out[name + "_bf16_256MiB"] = {"busbw_GBps": round(busbw(coll, S, t, R), 2), "ms": round(t * 1e3, 3),
                                      "instances": 32, "bit_exact": ok}
        for c, p in zip(comms, progs):
            c.unload(p)
        del send, recv
    return out


def run_multi(args, rank, world, local_rank):
    import torch
    if os.environ.get("MSCCL_FORCE_DEVICE"):  # testing the multi-process path on one GPU only
        local_rank = int(os.environ["MSCCL_FORCE_DEVICE"])
    import torch.distributed as dist
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
    torch.cuda.set_device(local_rank)
    if os.environ.get("MSCCL_FORCE_DEVICE"):  # NCCL refuses two ranks on one GPU; plumbing only anyway
        dist.init_process_group("gloo", rank=rank, world_size=world)
    else:
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", local_rank))
    set_params(rt, args)
    R = world
    algo = build_program(args, R)
    from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
    comm = mdist.init_from_process_group(local_rank)
    comm.load(algo.to_xml())
    S = int(args.size_mib * MIB)
    n = S // 2
    dev = torch.device("cuda", local_rank)
    send = synth.hashed(rank, torch.arange(n, device=dev, dtype=torch.int64), "bfloat16")
    recv = torch.empty(n, dtype=torch.bfloat16, device=dev)
    stream = torch.cuda.current_stream()
    for _ in range(args.warmup):
        comm.allreduce(send, recv, stream=stream)
    torch.cuda.synchronize()
    dist.barrier()
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
        comm.allreduce(send, recv, stream=stream)
    ev1.record(stream)
    torch.cuda.synchronize()
    dist.barrier()
    t = ev0.elapsed_time(ev1) / 1e3 / args.steps
    tt = torch.tensor([t], dtype=torch.float64)  # host tensor: works with any plumbing backend
    if dist.get_backend() == "nccl":
        tt = tt.to(dev)
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    t = float(tt.item())
    launches = rt.launch_count() - l0
    clk = clocks.stop() if clocks else None
    # sampled parity on this rank
    import numpy as np
    from oracle import irparse, sampled
    g = np.random.default_rng(1)
    idx = np.unique(g.integers(0, n, SEED_SAMPLES))
    want = sampled.allreduce_at(irparse.parse(algo.to_xml()), lambda r, i: synth.hashed_numpy(r, i, "bfloat16"),
                                n, "bfloat16", "sum", idx, rank=rank)
    got = recv[torch.from_numpy(idx).to(dev)].view(torch.int16).cpu().numpy().view(np.uint16)
    bad = torch.tensor([int(np.count_nonzero(got != want))])
    if dist.get_backend() == "nccl":
        bad = bad.to(dev)
    dist.all_reduce(bad)
    res = {"t": t, "launches": launches, "clocks": clk, "parity_bad": int(bad.item()),
           "parity_total": idx.size * R, "algo": algo, "S": S, "R": R}
    comm.destroy()
    dist.destroy_process_group()
    return res if rank == 0 else None


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
        if rank != 0:
            return
        R = world
    else:
        res = run_virtual(args)
        R = args.ranks
    S, t, algo = res["S"], res["t"], res["algo"]
    coll = res.get("coll", "allreduce")
    value = busbw(coll, S, t, R)
    peak, peak_src = measured_peak()
    per_chunk = S / algo.gpus[0].i_chunks
    nranks_launch = R if world == 1 else 1
    if "touches" in res:
        alg_bytes = sum(res["touches"]) * per_chunk
    else:
        alg_bytes = sum(simple_bytes_per_rank(algo, q, per_chunk) for q in range(R)) / R * nranks_launch
    launches_per_step = max(1, res["launches"] // args.steps)
    achieved = alg_bytes / t / 1e9
    traffic, prof = ncu_traffic()
    if world > 1:
        # one rank per GPU: the ring's bytes cross NVLink; roofline = measured peer copy 770 GB/s
        # per direction (B200_PROFILING.md; 900 nominal). Egress per rank per step = busBW * t.
        roof = {"bound": "nvlink", "achieved": round(value, 1), "peak": 770.0, "unit": "GB/s",
                "frac": round(value / 770.0, 4), "traffic": None,
                "peak_source": "measured peer copy per direction (B200_PROFILING.md)",
                "kernel": "mscclInterpreter<bf16,sum>", "algorithmic_bytes_per_launch": int(S * 2 * (R - 1) / R),
                "launch_ms": round(t * 1e3 / launches_per_step, 4)}
    else:
        # All R ranks run in one launch on one GPU: the HBM bytes any implementation must move are
        # every rank's input read once and its output written once.
        launch_s = t / launches_per_step
        compulsory = 2 * S * R
        hbm_achieved = compulsory / launch_s / 1e9
        l2peak, l2src = l2_peak()
        is_default = (args.program, args.instances, args.channels, args.slot_kib, args.threads, args.protocol) == \
            ("ring", 32, 1, 256, 256, "Simple")
        roof = {"bound": "hbm", "achieved": round(hbm_achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(hbm_achieved / peak, 4), "traffic": traffic if is_default else None,
                "peak_source": peak_src,
                "kernel": "mscclInterpreter<bf16,%s,Simple>" % ("copy" if coll == "alltoall" else "sum"),
                "algorithmic_bytes_per_launch": int(compulsory), "launch_ms": round(launch_s * 1e3, 4),
                "note": "algorithmic = compulsory HBM bytes of one launch covering all %d ranks: every input read "
                        "once + every output written once (2 S R); traffic = ncu dram read+write bytes per launch "
                        "(profiles/ncu_summary.json, default config only)" % R,
                "l2": {"touched_bytes_per_launch": int(alg_bytes), "achieved": round(achieved, 1),
                       "peak": l2peak, "frac": round(achieved / l2peak, 4) if l2peak else None,
                       "peak_source": l2src,
                       "note": "touched = the program's per-instruction operand bytes (send 2, recv 2, copy 2, "
                               "reduce/rrc/rrs 3, rrcs 4, rcs 3 chunks; a direct recv 0, a direct rcs 2), i.e. "
                               "the L2-level traffic of the interpreter; FIFO slots live mostly in L2"},
                "direct_placement": res.get("direct")}
    out = {
        "metric": metric_name(coll), "value": round(value, 3), "unit": "GB/s", "n_gpus": N,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 4),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
        "data": "synthetic (counter-based uniform[-1,1) bf16, seed 20230325+rank)",
        "config": config_dict(args, R, N),
        "frac_nvlink": round(value / 900.0, 4),
        "roofline": roof,
        "gpu_launches": res["launches"],
        "parity": {"sampled_outputs": res["parity_total"], "mismatches": res["parity_bad"],
                   "against": "oracle reduction trees (oracle/sampled.py), bit-exact"},
        "clocks": res["clocks"],
    }
    if "e2e" in res:
        out["e2e"] = res["e2e"]
    if "extras" in res:
        out["extras"] = res["extras"]
    if world == 1 and not args.no_cpu:
        out["cpu_baseline"] = cpu_oracle_run(args, R, algo, 32 * MIB)
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
