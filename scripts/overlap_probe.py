"""Does H2D of step k+1 overlap D2H of step k?  Pure torch streams + events, 31 chunks of 130 MB,
a busy-wait kernel stands in for each gridder/degridder group (1.5 ms)."""
import torch, time
nch, chunk = 31, 130 << 20
hin = torch.empty(nch * chunk, dtype=torch.uint8, pin_memory=True)
hout = torch.empty(nch * chunk, dtype=torch.uint8, pin_memory=True)
din = torch.empty(nch * chunk, dtype=torch.uint8, device="cuda")
dout = torch.empty(nch * chunk, dtype=torch.uint8, device="cuda")
s_h2d, s_d2h = torch.cuda.Stream(), torch.cuda.Stream()
comp = torch.cuda.current_stream()
ev_in = [torch.cuda.Event() for _ in range(nch)]
ev_k = [torch.cuda.Event() for _ in range(nch)]
ev_out = [torch.cuda.Event() for _ in range(nch)]
cycles = int(1.5e-3 * 1.9e9)
def step():
    for b in range(nch):
        s_h2d.wait_event(ev_k[b])
        with torch.cuda.stream(s_h2d):
            din[b*chunk:(b+1)*chunk].copy_(hin[b*chunk:(b+1)*chunk], non_blocking=True)
        ev_in[b].record(s_h2d)
        comp.wait_event(ev_in[b])
        torch.cuda._sleep(cycles)
        ev_k[b].record(comp)
    for b in range(nch):
        comp.wait_event(ev_out[b])
        torch.cuda._sleep(cycles)
        ev_k[b].record(comp)
        s_d2h.wait_event(ev_k[b])
        with torch.cuda.stream(s_d2h):
            hout[b*chunk:(b+1)*chunk].copy_(dout[b*chunk:(b+1)*chunk], non_blocking=True)
        ev_out[b].record(s_d2h)
step(); torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(6): step()
torch.cuda.synchronize()
print(f"pattern: {(time.perf_counter()-t0)/6*1e3:.1f} ms per step (8 GB moved; 93 ms of 'kernels')")
