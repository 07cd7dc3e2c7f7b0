"""Decompose the 1 KiB one-shot AllReduce latency into its parts (8 virtual ranks, fp16,
CUDA-graph replay), with hand-written probe programs that each add one stage:

  nop        every rank one nop (launch + prologue + epilogue: the floor)
  hop        rank r -> r+1, one LL message
  scatter    one-shot phase 1 only: every rank's input into every peer's scratch (7 sends,
             7 receives per rank)
  scatter+d  the same, receives set hasdep and one more block waits on all seven (nop)
  fold       one block per rank folds in + 7 scratch chunks into out (no communication)
  oneshot    the shipped one-shot program

Usage: python tools/latprobe.py [--proto LL] [--iters 200]   (needs a GPU)
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _step(s, typ, sb="-", so=-1, db="-", do=-1, depid="-1", deps="-1", hasdep=0):
    return ('<step s="%d" type="%s" srcbuf="%s" srcoff="%d" dstbuf="%s" dstoff="%d" cnt="1" depid="%s" deps="%s" '
            'hasdep="%d"/>' % (s, typ, sb, so, db, do, depid, deps, hasdep))


def _algo(name, R, proto, gpus):
    return '<algo name="%s" coll="custom" ngpus="%d" proto="%s" inplace="0" nchannels="1">%s</algo>' % (
        name, R, proto, "".join(gpus))


def scatter_ir(R, proto, with_dep):
    gpus = []
    for q in range(R):
        tbs = []
        peers = [p for p in range(R) if p != q]
        for p in peers:
            tbs.append('<tb id="%d" send="%d" recv="-1" chan="0">%s</tb>' % (len(tbs), p, _step(0, "s", "i", 0)))
        first_recv = len(tbs)
        for p in peers:
            tbs.append('<tb id="%d" send="-1" recv="%d" chan="0">%s</tb>' % (
                len(tbs), p, _step(0, "r", db="s", do=p, hasdep=1 if with_dep else 0)))
        if with_dep:
            ids = ",".join(str(first_recv + k) for k in range(len(peers)))
            zeros = ",".join("0" for _ in peers)
            tbs.append('<tb id="%d" send="-1" recv="-1" chan="0">%s</tb>' % (len(tbs), _step(0, "nop", depid=ids,
                                                                                             deps=zeros)))
        gpus.append('<gpu id="%d" i_chunks="1" o_chunks="1" s_chunks="%d">%s</gpu>' % (q, R, "".join(tbs)))
    return _algo("scatter", R, proto, gpus)


def fold_ir(R, proto, members=None, repeat=1):
    """one block per rank: cpy in -> out, then `members`-1 reduces of scratch chunks into out
    (a fused chain, reading R16); members = R is the one-shot fold; `repeat` runs the same
    chain again in the same block (warm instruction cache, same data)"""
    members = R if members is None else members
    gpus = []
    for q in range(R):
        steps = []
        for _ in range(repeat):
            steps.append(_step(len(steps), "cpy", "i", 0, "o", 0))
            k = 1
            for p in range(R):
                if p != q and k < members:
                    steps.append(_step(len(steps), "re", "s", p, "o", 0))
                    k += 1
        gpus.append('<gpu id="%d" i_chunks="1" o_chunks="1" s_chunks="%d"><tb id="0" send="-1" recv="-1" chan="0">'
                    '%s</tb></gpu>' % (q, R, "".join(steps)))
    return _algo("fold", R, proto, gpus)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--proto", default="LL")
    ap.add_argument("--iters", type=int, default=200)
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--n", type=int, default=512, help="fp16 elements per rank (512 = 1 KiB)")
    args = ap.parse_args()
    import torch
    import bench
    import synth
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
    W = args.ranks
    dev = torch.device("cuda:0")
    comms = rt.Comm.virtual(W, 0)
    R = bench.Ranks(rt, comms, list(range(W)), W, 1, dev)
    stream = torch.cuda.current_stream()
    n = args.n
    send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(W)]
    recv = [torch.empty_like(x) for x in send]
    probes = [("nop", bench.nop_ir(W)), ("hop", bench.hop_ir(W, args.proto)),
              ("scatter", scatter_ir(W, args.proto, False)), ("scatter+d", scatter_ir(W, args.proto, True)),
              ("copy", fold_ir(W, args.proto, 1)), ("fold2", fold_ir(W, args.proto, 2)),
              ("fold4", fold_ir(W, args.proto, 4)), ("fold", fold_ir(W, args.proto)),
              ("copy_x2", fold_ir(W, args.proto, 1, 2)), ("fold_x2", fold_ir(W, args.proto, None, 2)),
              ("fold_x4", fold_ir(W, args.proto, None, 4)),
              ("oneshot", P.oneshot_allreduce(W, protocol=args.proto).to_xml()),
              ("nvls", P.nvls_allreduce(W, 1).to_xml())]
    out = {"proto": args.proto, "ranks": W, "bytes": 2 * n, "mode": None}
    for name, ir in probes:
        progs = [c.load(ir) for c in comms]
        try:
            t, mode = bench.timed(lambda: R.call(progs, send, recv, n), args.iters, 10, stream, True, R)
            out[name] = round(t * 1e6, 2)
            out["mode"] = mode
        except Exception as e:
            out[name] = "error: %s" % str(e)[:200]
        R.unload(progs)
    print(json.dumps(out))
    for c in comms:
        c.destroy()


if __name__ == "__main__":
    main()
