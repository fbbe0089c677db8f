"""Helpers for GPU tests: run the CUDA path (through the C ABI) on a Workload."""
import numpy as np


def gpu_models(w, device=0):
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    return syn.Model(w.speedup, device), syn.Model(w.energy, device), syn.Clocks(w.freqs, device)


def gpu_sweep(w, want_pred=False, models=None):
    import torch
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    sp, en, ck = models or gpu_models(w)
    feats = torch.from_numpy(np.ascontiguousarray(w.features)).cuda()
    S = E = None
    if want_pred:
        S = torch.empty((w.n_kernels, w.n_freqs), dtype=torch.float32, device="cuda")
        E = torch.empty_like(S)
    ch = syn.sweep(sp, en, feats, ck, w.default_idx, w.targets, out_speedup=S, out_energy=E)
    torch.cuda.synchronize()
    out = {"choice": ch.cpu().numpy()}
    if want_pred:
        out["S"], out["E"] = S.cpu().numpy(), E.cpu().numpy()
    return out


def gpu_predict(w, default_idx=None, models=None):
    import torch
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    sp, en, ck = models or gpu_models(w)
    feats = torch.from_numpy(np.ascontiguousarray(w.features)).cuda()
    S, E = syn.predict(sp, en, feats, ck, w.default_idx if default_idx is None else default_idx)
    torch.cuda.synchronize()
    return S.cpu().numpy(), E.cpu().numpy()


def assert_bits_equal(a, b, what):
    """Bit-exact fp32 comparison (NaNs compare by bits too)."""
    a = np.ascontiguousarray(a, np.float32).view(np.uint32)
    b = np.ascontiguousarray(b, np.float32).view(np.uint32)
    bad = np.flatnonzero(a.reshape(-1) != b.reshape(-1))
    assert bad.size == 0, f"{what}: {bad.size} mismatches, first at {bad[:5]}"


def assert_choices(gpu, ref, gap=None, tol=1e-5, what="choice"):
    """Choices bit-exact, except (north_star) where the oracle's best and runner-up keys differ by
    less than `tol` relative — counted and required to be zero here since predictions are exact."""
    diff = gpu != ref
    if gap is not None:
        exempt = diff & (gap < tol)
        assert not exempt.any(), f"{what}: {int(exempt.sum())} tolerance exemptions used"
    assert not diff.any(), f"{what}: {int(diff.sum())} mismatches, first at {np.argwhere(diff)[:5].tolist()}"
