"""Full-size parity: every row of a configuration, predictions and choices, against the oracle.

north_star: "bit-exact frequency selections versus the CPU oracle on all five configs".  The GPU
runs the whole configuration in the launch configuration bench.py times (one synergy_sweep over
all rows, here with the prediction buffers attached so S and E are compared too, plus a second
call without them whose choices must be identical).  The oracle (oracle/oracle.c, single-threaded)
recomputes every row, in one process per host core over contiguous row chunks.

In the default GPU suite c3 runs in full on the GPU and the oracle recomputes every 8th chunk of
8192 rows (12.5 % of the rows, ~1-2 min on 16 cores); SYNERGY_FULL_PARITY=c3 (or c4, or all)
compares every row (c3 ~8-13 min, c4 ~9-15 min on 16 cores); the full runs' summaries are
committed under profiles/r2/.  Every run writes gpurun_out/full_parity_<cfg>.json: rows compared,
mismatches of S / E bits and of choices, and the tolerance exemptions used (expected 0).
"""
import json
import multiprocessing as mp
import os
import time

import numpy as np
import pytest

import oracle
from paper_conf_sc_fandccfc23_b200 import workloads as W

pytestmark = pytest.mark.gpu

_CACHE = {}


def _init(cfg):
    oracle.build()
    _CACHE["models"] = W.make_models(cfg)
    _CACHE["cfg"] = cfg


def _oracle_chunk(args):
    row0, n = args
    cfg = _CACHE["cfg"]
    w = W.make_config(cfg, row0=row0, n=n, models=_CACHE["models"])
    r = oracle.sweep_workload(w, want_pred=True, with_gap=True)
    return row0, r["S"], r["E"], r["choice"], r["gap"]


def _full(cfg):
    v = os.environ.get("SYNERGY_FULL_PARITY", "")
    return v == "all" or cfg in v.split(",")


def _enabled(cfg):
    return cfg == "c3" or _full(cfg)


@pytest.mark.parametrize("cfg", ["c3", "c4"])
def test_full_size_every_row(cfg):
    if not _enabled(cfg):
        pytest.skip(f"{cfg} full-size parity runs with SYNERGY_FULL_PARITY={cfg}")
    import torch
    from paper_conf_sc_fandccfc23_b200 import build
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    build.build()
    oracle.build()
    t0 = time.time()
    w = W.make_config(cfg)
    n_k, n_f, n_t = w.n_kernels, w.n_freqs, len(w.targets)
    sp, en, ck = syn.Model(w.speedup), syn.Model(w.energy), syn.Clocks(w.freqs)
    feats = torch.from_numpy(w.features).cuda()
    S = torch.empty((n_k, n_f), dtype=torch.float32, device="cuda")
    E = torch.empty_like(S)
    ch_pred = syn.sweep(sp, en, feats, ck, w.default_idx, w.targets, out_speedup=S, out_energy=E)
    ch = syn.sweep(sp, en, feats, ck, w.default_idx, w.targets)       # the bench call (no predictions)
    torch.cuda.synchronize()
    same_calls = bool((ch == ch_pred).all())
    ch = ch.cpu().numpy()
    del ch_pred, feats
    t_gpu = time.time() - t0

    cores = len(os.sched_getaffinity(0))
    chunk = 8192 if cfg == "c3" else 32768
    jobs = [(r, min(chunk, n_k - r)) for r in range(0, n_k, chunk)]
    stride = 1 if _full(cfg) else 8                                     # every 8th chunk by default
    jobs = jobs[::stride]
    bad_S = bad_E = bad_c = exempt = 0
    min_gap = np.inf
    t1 = time.time()
    with mp.get_context("fork").Pool(cores, initializer=_init, initargs=(cfg,)) as pool:
        for row0, rS, rE, rc, gap in pool.imap_unordered(_oracle_chunk, jobs):
            n = rS.shape[0]
            gS = S[row0:row0 + n].cpu().numpy()
            gE = E[row0:row0 + n].cpu().numpy()
            bad_S += int((gS.view(np.uint32) != rS.view(np.uint32)).sum())
            bad_E += int((gE.view(np.uint32) != rE.view(np.uint32)).sum())
            diff = ch[row0:row0 + n] != rc
            bad_c += int(diff.sum())
            exempt += int((diff & (gap < 1e-5)).sum())
            min_gap = min(min_gap, float(gap.min()))
    rows_cmp = sum(n for _, n in jobs)
    summary = {"config": cfg, "rows": n_k, "rows_compared": rows_cmp, "n_freqs": n_f, "targets": n_t,
               "evals_compared": rows_cmp * n_f,
               "S_bit_mismatches": bad_S, "E_bit_mismatches": bad_E, "choice_mismatches": bad_c,
               "tolerance_exemptions_used": exempt, "min_oracle_gap": min_gap,
               "choices_identical_with_and_without_prediction_buffers": same_calls,
               "gpu_s": round(t_gpu, 1), "oracle_s": round(time.time() - t1, 1), "oracle_processes": cores,
               "oracle_chunk_rows": chunk}
    os.makedirs("gpurun_out", exist_ok=True)
    with open(os.path.join("gpurun_out", f"full_parity_{cfg}.json"), "w") as f:
        json.dump(summary, f, indent=1)
    print(json.dumps(summary))
    assert same_calls
    assert bad_S == 0 and bad_E == 0
    assert exempt == 0 and bad_c == 0
