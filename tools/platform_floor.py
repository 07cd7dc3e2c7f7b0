"""Platform launch floor for comparison with the interpreter's floor_nop (bench extras):
CUDA-graph replay of a trivial one-element torch kernel and of a cooperative launch of an
empty kernel (cuda-python driver API is not needed: torch + ctypes on libcudart)."""
import json
import torch

x = torch.zeros(1, device="cuda")
s = torch.cuda.Stream()
g = torch.cuda.CUDAGraph()
x.add_(1)
torch.cuda.synchronize()
with torch.cuda.graph(g, stream=s):
    for _ in range(50):
        x.add_(1)
g.replay()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20):
    g.replay()
e1.record()
torch.cuda.synchronize()
print(json.dumps({"graph_replay_trivial_kernel_us": round(e0.elapsed_time(e1) * 1e3 / (20 * 50), 3)}))
