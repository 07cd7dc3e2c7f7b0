"""Latency floor of the interpreter on 8 virtual ranks (CUDA-graph replay): a program whose
only instruction per rank is a local copy (no communication) vs the 1 KiB AllReduce programs."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, bench, synth
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime as rt
R = 8
rt.set_param("MSCCL_THREADS", int(os.environ.get("THREADS", 256)))


def local_ir(proto):
    out = ['<algo name="local" coll="allreduce" ngpus="%d" proto="%s" inplace="0" nchannels="1" ninstances="1">'
           % (R, proto)]
    for q in range(R):
        out.append('  <gpu id="%d" i_chunks="1" o_chunks="1" s_chunks="0">' % q)
        out.append('    <tb id="0" send="-1" recv="-1" chan="0">')
        out.append('      <step s="0" type="cpy" srcbuf="i" srcoff="0" dstbuf="o" dstoff="0" cnt="1" depid="-1" '
                   'deps="-1" hasdep="0"/>')
        out.append('    </tb>')
        out.append('  </gpu>')
    out.append('</algo>')
    return "\n".join(out)


comms = rt.Comm.virtual(R, 0)
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream()
n = 512
send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(R)]
recv = [torch.empty_like(x) for x in send]
cases = [("local_copy_LL", local_ir("LL")), ("local_copy_Simple", local_ir("Simple")),
         ("oneshot_LL", P.oneshot_allreduce(R, protocol="LL").to_xml()),
         ("allpairs_LL", P.allpairs_allreduce(R, protocol="LL").to_xml()),
         ("ring_ch8_LL", P.ring_allreduce(R, channels=8, protocol="LL").to_xml())]
for name, ir in cases:
    progs = [c.load(ir) for c in comms]

    def call():
        with rt.group():
            for q in range(R):
                comms[q].run(progs[q], send[q], recv[q], n)
    t, mode = bench._timed(call, 50, stream)
    te, _ = bench._timed(call, 50, stream, graph=False)
    print(json.dumps({"program": name, "us_graph": round(t * 1e6, 2), "us_eager": round(te * 1e6, 2),
                      "ctas": sum(p.info()["thread_blocks"] for p in progs)}), flush=True)
    for c, p in zip(comms, progs):
        c.unload(p)
