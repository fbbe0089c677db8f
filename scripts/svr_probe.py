"""Time the SVR path (k_svr_v + k_svr + finish) on config shapes: speedup linear, energy SVR."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_sc_fandccfc23_b200 import synergy as syn, workloads as W

for cfg in sys.argv[1:] or ["c2"]:
    n_k, n_f = W.CONFIGS[cfg][0], W.CONFIGS[cfg][1]
    freqs = W.clock_table(n_f)
    d = W.default_index(freqs)
    for n_sv in (512, 2048):
        sp = W.linear_speedup_model(np.random.SeedSequence(1), W.N_STATIC, freqs, d)
        en = W.svr_energy_model(np.random.SeedSequence(2), W.N_STATIC, freqs, d, n_sv=n_sv)
        feats = torch.from_numpy(W.make_features(cfg)).cuda()
        hs, he, ck = syn.Model(sp), syn.Model(en), syn.Clocks(freqs)
        ch = torch.empty((n_k, 6), dtype=torch.int32, device="cuda")
        for _ in range(3):
            syn.sweep(hs, he, feats, ck, d, W.targets_six(), out=ch)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 20
        a.record()
        for _ in range(reps):
            syn.sweep(hs, he, feats, ck, d, W.targets_six(), out=ch)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / reps
        flops = 2.0 * n_k * n_f * n_sv
        print(json.dumps({"cfg": cfg, "n_sv": n_sv, "ms": ms, "contraction_tflops": flops / ms / 1e9,
                          "launch": syn.last_launch()}))
