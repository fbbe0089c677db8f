"""Probe the scattered-load microbenchmark (tools/peaks.cu) over load widths and window sizes."""
import ctypes as C, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import tools
tools.build_peaks()
lib = C.CDLL(tools._PEAKS_SO)
lib.peaks_scatter.argtypes = [C.c_int, C.c_int, C.c_uint, C.c_int, C.c_void_p]
res = {"summary": tools.measure_peaks(0)}
for width in (32, 64, 128, 1):
    for win in (2048, 4096, 1 << 16):
        out = np.zeros(2)
        rc = lib.peaks_scatter(0, width, win, 1024, out.ctypes.data)
        res[f"w{width}_win{win}"] = {"rc": rc, "GB_s": out[0] / 1e9, "Gloads_s": out[1] / 1e9,
                                     "loads_per_clk_sm_at_1965": out[1] / 148 / 1.965e9}
print(json.dumps(res, indent=1))
