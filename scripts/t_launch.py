import torch
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
y = torch.zeros(1024, device="cuda")
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
g = torch.cuda.CUDAGraph()
st = torch.cuda.Stream()
with torch.cuda.stream(st):
    y.add_(1); torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=st):
        y.add_(1)
for label, fl in (("flushed", True), ("no flush", False)):
    ts = []
    for _ in range(30):
        torch.cuda.synchronize()
        if fl: flush.zero_()
        s.record(); g.replay(); e.record(); torch.cuda.synchronize()
        ts.append(s.elapsed_time(e) * 1e3)
    print(label, "trivial kernel graph replay: median %.2f us min %.2f" % (sorted(ts)[15], min(ts)))
