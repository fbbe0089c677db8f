"""Per-call device time with events vs kernel durations (diagnostic)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_fandccfc23_b200 import synergy as syn, workloads as W
cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
w = W.make_config(cfg)
sp, en, ck = syn.Model(w.speedup, 0), syn.Model(w.energy, 0), syn.Clocks(w.freqs, 0)
f = torch.from_numpy(w.features).cuda()
out = torch.empty((w.n_kernels, len(w.targets)), dtype=torch.int32, device="cuda")
ref = None
st = torch.cuda.current_stream()
ts = []
for i in range(12):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(st)
    syn.sweep(sp, en, f, ck, w.default_idx, w.targets, out=out)
    b.record(st)
    torch.cuda.synchronize()
    ts.append(a.elapsed_time(b) * 1e3)
    o = out.cpu()
    if ref is None: ref = o.clone()
    elif not torch.equal(o, ref): print("call", i, "DIFFERS from call 0:", int((o != ref).sum()), "entries")
print(cfg, "ILV", os.environ.get("SYNERGY_TM_ILV", "auto"), "per-call us:", [round(x, 1) for x in ts])
