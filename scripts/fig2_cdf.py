"""Fig. 2 analogue: CDF of the block relative value
range (block max - min over the global range, oracle/analytics.py) for b = 8..128 on the
synthetic fields.  One JSON line per (field, b) with the CDF at fixed thresholds."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import synth
from oracle import analytics as A

FIELDS = {
    "cesm_T": lambda: synth.cesm_like(0).numpy(),
    "cesm_cloud": lambda: synth.cesm_like(1).numpy(),
    "hurricane_U": lambda: synth.hurricane_like(0).numpy(),
    "hurricane_QSNOW": lambda: synth.hurricane_like(1).numpy(),
    "nyx_density": lambda: synth.nyx_like(0, n=256).numpy(),
    "nyx_velocity": lambda: synth.nyx_like(1, n=256).numpy(),
    "nyx_temperature": lambda: synth.nyx_like(2, n=256).numpy(),
    "hacc_velocity": lambda: synth.hacc_like(0, n=20_000_000).numpy(),
    "hacc_position": lambda: synth.hacc_like(1, n=20_000_000).numpy(),
    "miranda_f64": lambda: synth.miranda_like().numpy(),
    "qmcpack_f64": lambda: synth.qmcpack_like().numpy(),
}
TH = [1e-4, 1e-3, 1e-2, 3e-2, 1e-1, 3e-1, 1.0]
for name, gen in FIELDS.items():
    x = np.ascontiguousarray(gen()).reshape(-1)
    for b in (8, 16, 32, 64, 128):
        r = A.block_relative_range(x, b)
        print(json.dumps({"field": name, "n": int(x.size), "block": b, "blocks": int(r.size),
                          "thresholds": TH, "cdf": A.cdf_points(r, TH),
                          "median_rel_range": float(np.median(r)) if r.size else None}), flush=True)
