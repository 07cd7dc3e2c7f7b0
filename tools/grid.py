"""BASELINE configs[2] and configs[4] as measured grids on virtual ranks (one B200):

  c3: all-pairs (two-shot) and one-shot AllReduce, fp16, LL, instances r in {1, 2, 4},
      1 KiB .. 4 MiB per rank (x4 steps): CUDA-graph time per op;
  c5: ring AllGather and ReduceScatter, bf16, Simple, R in {2, 4, 8} x r in {1, 2, 4},
      1 MiB / 16 MiB / 256 MiB per rank: busBW.

Each point: 20 warm-up + 50 timed ops (20 at 256 MiB) under CUDA-graph replay (bench.timed),
plus a correctness check of the last op (exact for AllGather, sampled oracle reduction trees
for AllReduce / ReduceScatter). Writes JSON lines to argv[1] (default
gpurun_out/grid.jsonl) and prints a markdown table.

Usage: python tools/grid.py [out.jsonl]   (needs a GPU)
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

MIB = 1 << 20


def main():
    import torch
    import bench
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
    out_path = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "grid.jsonl")
    os.makedirs(os.path.dirname(out_path), exist_ok=True)
    f = open(out_path, "w")
    rt.set_param("MSCCL_TIMEOUT_S", 60)
    rt.set_param("MSCCL_MAX_CHANNELS", 64)
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream()
    rows = []

    def emit(rec):
        rows.append(rec)
        f.write(json.dumps(rec) + "\n")
        f.flush()
        print(json.dumps(rec), flush=True)

    # ---- c3: all-pairs / one-shot AllReduce, fp16, LL
    W = 8
    comms = rt.Comm.virtual(W, 0)
    R = bench.Ranks(rt, comms, list(range(W)), W, 1, dev)
    for name, build in (("allpairs", lambda r: P.allpairs_allreduce(W, r, protocol="LL")),
                        ("oneshot", lambda r: P.oneshot_allreduce(W, 1, r, protocol="LL"))):
        for r in (1, 2, 4):
            algo = build(r)
            try:
                progs = R.load(algo, 0, 0)
            except Exception as e:   # e.g. more thread blocks than fit co-resident
                emit({"config": "c3", "program": name, "instances": r, "error": str(e)[:160]})
                continue
            size = 1024
            while size <= 4 * MIB:
                n = size // 2
                send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(W)]
                recv = [torch.empty_like(x) for x in send]
                try:
                    t, mode = bench.timed(lambda: R.call(progs, send, recv, n), 50, 20, stream, True, R)
                    bad, _ = bench.sampled_parity(algo, recv, n, [0, W - 1], local=list(range(W)), dtype="float16")
                    emit({"config": "c3", "coll": "allreduce", "program": algo.name, "R": W, "instances": r,
                          "dtype": "fp16", "proto": "LL", "bytes": size, "t_us": round(t * 1e6, 2),
                          "busbw": round(bench.busbw("allreduce", size, t, W), 3), "mode": mode,
                          "correct": bad == 0})
                except Exception as e:
                    emit({"config": "c3", "program": algo.name, "bytes": size, "error": str(e)[:160]})
                del send, recv
                size *= 4
            R.unload(progs)
    for c in comms:
        c.destroy()

    # ---- c5: ring AllGather / ReduceScatter, bf16, Simple, R x instances
    for W in (2, 4, 8):
        comms = rt.Comm.virtual(W, 0)
        R = bench.Ranks(rt, comms, list(range(W)), W, 1, dev)
        for coll in ("allgather", "reducescatter"):
            for r in (1, 2, 4):
                algo = P.ring_allgather(W, 1, r) if coll == "allgather" else P.ring_reducescatter(W, 1, r)
                progs = R.load(algo, 0, 0)
                for S in (1 * MIB, 16 * MIB, 256 * MIB):
                    n = S // 2                      # elements of the larger buffer per rank
                    ns, nr, count = bench.shapes(coll, n, W)
                    send = [synth.hashed(q, torch.arange(ns, device=dev, dtype=torch.int64), "bfloat16")
                            for q in range(W)]
                    recv = [torch.empty(nr, dtype=torch.bfloat16, device=dev) for _ in range(W)]
                    iters = 20 if S >= 256 * MIB else 50
                    try:
                        t, mode = bench.timed(lambda: R.call(progs, send, recv, count), iters, 20, stream, True, R)
                        if coll == "allgather":
                            ok = bench.check_allgather(R, recv, W, count)
                        else:
                            bad, _ = bench.sampled_parity(algo, recv, count, [0, W - 1], local=list(range(W)))
                            ok = bad == 0
                        emit({"config": "c5", "coll": coll, "program": algo.name, "R": W, "instances": r,
                              "dtype": "bf16", "proto": "Simple", "bytes": S, "t_us": round(t * 1e6, 2),
                              "busbw": round(bench.busbw(coll, S, t, W), 3), "mode": mode, "correct": bool(ok)})
                    except Exception as e:
                        emit({"config": "c5", "program": algo.name, "bytes": S, "error": str(e)[:160]})
                    del send, recv
                    torch.cuda.empty_cache()
                R.unload(progs)
        for c in comms:
            c.destroy()
    f.close()

    # markdown summary
    print("\n### c3: AllReduce fp16 LL, 8 virtual ranks, CUDA graph (us per op)\n")
    print("| bytes/rank | " + " | ".join("%s r=%d" % (p, r) for p in ("allpairs", "oneshot") for r in (1, 2, 4)) + " |")
    print("|---" * 7 + "|")
    sizes = sorted({x["bytes"] for x in rows if x.get("config") == "c3" and "t_us" in x})
    for sz in sizes:
        cells = []
        for p in ("allpairs", "oneshot"):
            for r in (1, 2, 4):
                hit = [x for x in rows if x.get("config") == "c3" and x.get("bytes") == sz and "t_us" in x
                       and x["program"].startswith(p) and x["instances"] == r]
                cells.append("%.1f%s" % (hit[0]["t_us"], "" if hit[0]["correct"] else " X") if hit else "-")
        print("| %d | %s |" % (sz, " | ".join(cells)))
    print("\n### c5: ring AllGather / ReduceScatter bf16, busBW GB/s (virtual ranks, HBM-bound)\n")
    print("| coll | R | r | 1 MiB | 16 MiB | 256 MiB |")
    print("|---|---|---|---|---|---|")
    for coll in ("allgather", "reducescatter"):
        for W in (2, 4, 8):
            for r in (1, 2, 4):
                cells = []
                for S in (1 * MIB, 16 * MIB, 256 * MIB):
                    hit = [x for x in rows if x.get("config") == "c5" and x.get("coll") == coll and x["R"] == W
                           and x["instances"] == r and x["bytes"] == S and "busbw" in x]
                    cells.append("%.1f%s" % (hit[0]["busbw"], "" if hit[0]["correct"] else " X") if hit else "-")
                print("| %s | %d | %d | %s |" % (coll, W, r, " | ".join(cells)))


if __name__ == "__main__":
    main()
