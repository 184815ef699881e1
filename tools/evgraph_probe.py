import torch
x = torch.randn(1<<24, device='cuda')
s = torch.cuda.Stream()
evs = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
g = torch.cuda.CUDAGraph()
s.wait_stream(torch.cuda.current_stream())
try:
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            evs[0].record(s); y = x * 2; evs[1].record(s); z = y + 1; evs[2].record(s)
    torch.cuda.synchronize(); g.replay(); torch.cuda.synchronize()
    print("events in graph OK", evs[0].elapsed_time(evs[1]), evs[1].elapsed_time(evs[2]))
except Exception as e:
    print("events in graph FAILED", repr(e)[:300])
