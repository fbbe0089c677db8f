"""Finish-phase probe: per-kernel times of sweep (predict+select) vs predict-only on a config,
and the standalone select on the resulting predictions.  Diagnostic only."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_fandccfc23_b200 import synergy as syn, workloads as W

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
K = 30
w = W.make_config(cfg)
sp, en, ck = syn.Model(w.speedup), syn.Model(w.energy), syn.Clocks(w.freqs)
feats = torch.from_numpy(w.features).cuda()
S = torch.empty((w.n_kernels, w.n_freqs), dtype=torch.float32, device="cuda")
E = torch.empty_like(S)
out = torch.empty((w.n_kernels, len(w.targets)), dtype=torch.int32, device="cuda")
flush = torch.empty(128 << 20, dtype=torch.float32, device="cuda")

def per_kernel(fn):
    for _ in range(3):
        flush.zero_(); fn()
    torch.cuda.synchronize(); syn.timing_read(); syn.timing_enable(True)
    for _ in range(K):
        flush.zero_(); fn()
    torch.cuda.synchronize(); syn.timing_enable(False)
    return {k: round(v[0] / max(v[1], 1) * 1e3, 2) for k, v in syn.timing_read().items()}

res = {"sweep_us": per_kernel(lambda: syn.sweep(sp, en, feats, ck, w.default_idx, w.targets, out=out)),
       "sweep_with_pred_us": per_kernel(lambda: syn.sweep(sp, en, feats, ck, w.default_idx, w.targets, out=out,
                                                          out_speedup=S, out_energy=E)),
       "predict_us": per_kernel(lambda: syn.predict(sp, en, feats, ck, w.default_idx, out_speedup=S, out_energy=E)),
       "select_us": per_kernel(lambda: syn.select(S, E, w.default_idx, w.targets, out=out))}
print(json.dumps({"cfg": cfg, **res}))
