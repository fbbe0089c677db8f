"""Host vs device time per sweep call (diagnostic): wall clock of the C-ABI call, event time."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_fandccfc23_b200 import synergy as syn, workloads as W
cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
w = W.make_config(cfg)
sp, en, ck = syn.Model(w.speedup, 0), syn.Model(w.energy, 0), syn.Clocks(w.freqs, 0)
f = torch.from_numpy(w.features).cuda()
out = torch.empty((w.n_kernels, len(w.targets)), dtype=torch.int32, device="cuda")
for _ in range(5):
    syn.sweep(sp, en, f, ck, w.default_idx, w.targets, out=out)
torch.cuda.synchronize()
st = torch.cuda.current_stream()
for rep in range(3):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    a.record(st)
    for _ in range(20):
        syn.sweep(sp, en, f, ck, w.default_idx, w.targets, out=out)
    b.record(st)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"{cfg} ILV={os.environ.get('SYNERGY_TM_ILV','auto')} host {1e6*(t1-t0)/20:.1f} us/call, device {1e3*a.elapsed_time(b)/20:.1f} us/call")

if "--prof" in sys.argv:
    from torch.profiler import profile, ProfilerActivity
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(10):
            syn.sweep(sp, en, f, ck, w.default_idx, w.targets, out=out)
        torch.cuda.synchronize()
    evs = [e for e in prof.events() if e.device_type.name == "CUDA"]
    evs.sort(key=lambda e: e.time_range.start)
    last = None
    for e in evs[:12]:
        gap = (e.time_range.start - last) if last is not None else 0
        print(f"{e.name[:40]:40s} start+{gap:8.1f} dur {e.time_range.end - e.time_range.start:8.1f} us")
        last = e.time_range.end
