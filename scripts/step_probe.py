"""Where does a c2 step's time go beyond the two kernels?  Times K steps (L2 flushed, CUDA events
on the launch stream) three ways: library timing events on, off, and the sweep replayed from a
CUDA graph.  Diagnostic only (not a bench line)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_fandccfc23_b200 import synergy as syn, workloads as W

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
K = 50
w = W.make_config(cfg)
sp, en, ck = syn.Model(w.speedup), syn.Model(w.energy), syn.Clocks(w.freqs)
feats = torch.from_numpy(w.features).cuda()
out = torch.empty((w.n_kernels, len(w.targets)), dtype=torch.int32, device="cuda")
flush = torch.empty(128 << 20, dtype=torch.float32, device="cuda")
st = torch.cuda.current_stream()

def run(fn, timing):
    syn.timing_enable(timing)
    for _ in range(5):
        flush.zero_(); fn()
    torch.cuda.synchronize()
    syn.timing_read()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for i in range(K):
        flush.zero_()
        ev[i][0].record(st); fn(); ev[i][1].record(st)
    torch.cuda.synchronize()
    kt = syn.timing_read()
    syn.timing_enable(False)
    ms = sorted(a.elapsed_time(b) for a, b in ev)
    return {"median_ms": ms[K // 2], "min_ms": ms[0], "kernels": {k: v[0] / max(v[1], 1) for k, v in kt.items()}}

sweep = lambda: syn.sweep(sp, en, feats, ck, w.default_idx, w.targets, out=out)
res = {"timing_on": run(sweep, True), "timing_off": run(sweep, False)}
g = torch.cuda.CUDAGraph()
s2 = torch.cuda.Stream()
s2.wait_stream(st)
with torch.cuda.stream(s2):
    sweep(); torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s2):
        sweep()
torch.cuda.synchronize()
res["graph"] = run(g.replay, False)
print(json.dumps({"cfg": cfg, **res}))
