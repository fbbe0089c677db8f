"""Product-path workloads for compute-sanitizer runs (memcheck / racecheck / synccheck / initcheck).

    compute-sanitizer --tool memcheck python scripts/sanitize_cases.py [small|full]

Exercises every library kernel through the C ABI on seeded inputs (no oracle: the sanitizer's
report is the result).  `small` (racecheck, the slowest tool) runs c1 and small fuzz shapes;
`full` adds c2, the slab pipeline, two streams and a CUDA-graph replay.
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_fandccfc23_b200 import synergy as syn  # noqa: E402
from paper_conf_sc_fandccfc23_b200 import workloads as W  # noqa: E402


def run(w, out_pred=True, stream=None):
    sp, en, ck = syn.Model(w.speedup), syn.Model(w.energy), syn.Clocks(w.freqs)
    f = torch.from_numpy(np.ascontiguousarray(w.features)).cuda()
    S = E = None
    if out_pred:
        S = torch.empty((w.n_kernels, w.n_freqs), dtype=torch.float32, device="cuda")
        E = torch.empty_like(S)
    ch = syn.sweep(sp, en, f, ck, w.default_idx, w.targets, out_speedup=S, out_energy=E, stream=stream)
    if w.n_kernels:
        S2, E2 = syn.predict(sp, en, f, ck, w.default_idx, stream=stream)
        syn.select(S2, E2, w.default_idx, w.targets, stream=stream)
        syn.pareto(S2, E2, stream=stream)
        syn.choice_error(S2, E2, w.default_idx, w.targets, ch, stream=stream)
        syn.plan(ch, ck, stream=stream)
    torch.cuda.synchronize()
    return ch


def main():
    mode = sys.argv[1] if len(sys.argv) > 1 else "full"
    cases = [W.make_config("c1"),
             W.fuzz_workload(1001, 3, 2, F=4, n_trees=3, max_depth=4),
             W.fuzz_workload(1002, 7, 31, F=5, n_trees=4, max_depth=6, exact_thresholds=True),
             W.fuzz_workload(1003, 11, 97, F=7, n_trees=6, max_depth=5, linear="both"),
             W.fuzz_workload(1004, 23, 196, F=4, n_trees=5, max_depth=14, p_freq=0.9, p_leaf=0.05)]
    if mode == "full":
        cases += [W.make_config("c2"), W.fuzz_workload(1005, 600, 64, F=5, n_trees=4, max_depth=9, linear="both")]
    cases.append(W.make_config("c1", models=W.make_models_svr("c1", n_sv=100, ensemble=True)))
    cases.append(W.fuzz_workload(1007, 9, 33, F=3, n_trees=4, max_depth=5, linear="only"))
    for w in cases:
        run(w)
        print("ok", w.name, w.n_kernels, w.n_freqs, flush=True)
    syn.config_set("svr_tc", 0)                              # the fp64 SVR reference path too
    run(W.make_config("c1", models=W.make_models_svr("c1", n_sv=100)))
    syn.config_set("svr_tc", 1)
    syn.config_set("algo", 1)                                # the general exact path on c1
    run(W.make_config("c1"))
    syn.config_set("algo", 0)
    print("ok svr fp64 + general path", flush=True)
    syn.config_set("tm_small", 0)                            # c1 on the two-kernel walk path too
    run(W.make_config("c1"))
    syn.config_set("tm_small", 1)                            # and the single-launch path on a fuzz case
    run(W.fuzz_workload(1008, 40, 70, F=6, n_trees=5, max_depth=9, linear="both"))
    syn.config_set("tm_small", -1)
    print("ok walk / single-launch paths", flush=True)
    if mode == "full":
        syn.config_set("tm_slab", 64)
        syn.config_set("tm_kb", 32)
        w = W.fuzz_workload(1006, 300, 128, F=12, n_trees=3, max_depth=6)
        run(w)
        print("ok slab pipeline", flush=True)
        syn.config_set("tm_slab", 0)
        for kb in (512, 1024):                               # the large-batch block shapes
            syn.config_set("tm_kb", kb)
            syn.config_set("tm_nt", 1024)
            run(W.make_config("c2"))
            print("ok kb", kb, flush=True)
        syn.config_set("tm_kb", 0)
        syn.config_set("tm_nt", 0)
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        w = W.make_config("c1")
        with torch.cuda.stream(s1):
            run(w, stream=s1)
        with torch.cuda.stream(s2):
            run(w, stream=s2)
        torch.cuda.synchronize()
        print("ok two streams", flush=True)
    print("SANITIZE_CASES_DONE", flush=True)


if __name__ == "__main__":
    main()
