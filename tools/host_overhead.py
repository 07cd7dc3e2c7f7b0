"""Host-side cost of one 8-rank group call through the Python binding and the C ABI."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import cProfile, pstats
import torch, synth
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime as rt
R = 8
comms = rt.Comm.virtual(R, 0)
dev = torch.device("cuda:0")
n = 512
send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(R)]
recv = [torch.empty_like(x) for x in send]
progs = [c.load(P.ring_allreduce(R, channels=8, protocol="LL").to_xml()) for c in comms]
stream = torch.cuda.current_stream()


def call():
    with rt.group():
        for q in range(R):
            comms[q].run(progs[q], send[q], recv[q], n, stream=stream)


for _ in range(100):
    call()
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(2000):
    call()
t1 = time.perf_counter()
torch.cuda.synchronize()
t2 = time.perf_counter()
print("host enqueue per group call: %.1f us; incl. drain %.1f us" % ((t1 - t0) / 2000 * 1e6, (t2 - t0) / 2000 * 1e6))
pr = cProfile.Profile()
pr.enable()
for _ in range(500):
    call()
pr.disable()
torch.cuda.synchronize()
pstats.Stats(pr).sort_stats("tottime").print_stats(12)
