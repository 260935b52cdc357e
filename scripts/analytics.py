"""SURVEY 8(f) row 1 analytics on the synthetic fields (oracle side, CPU):
Formula 6 shift overhead (Solution C vs A/B; the Fig. 6
analogue) and Formula 7 PSNR / max error per field and block size (8 and 16
are oracle-only points of the Fig. 8 block-size study), at the
small shapes the oracle finishes in seconds.  Writes one JSON line per
(field, eb, b) to stdout."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import oracle
import synth

FIELDS = {
    "cesm_T": lambda: synth.cesm_like(0, shape=(450, 900)).numpy(),
    "cesm_cloud": lambda: synth.cesm_like(1, shape=(450, 900)).numpy(),
    "hurricane_U": lambda: synth.hurricane_like(0, shape=(25, 125, 125)).numpy(),
    "hurricane_QSNOW": lambda: synth.hurricane_like(1, shape=(25, 125, 125)).numpy(),
    "nyx_density": lambda: synth.nyx_like(0, n=96).numpy(),
    "nyx_velocity": lambda: synth.nyx_like(1, n=96).numpy(),
    "nyx_temperature": lambda: synth.nyx_like(2, n=96).numpy(),
    "hacc_velocity": lambda: synth.hacc_like(0, n=1_000_003).numpy(),
    "hacc_position": lambda: synth.hacc_like(1, n=1_000_003).numpy(),
    "miranda_f64": lambda: synth.miranda_like(shape=(64, 96, 96)).numpy(),
}

for name, gen in FIELDS.items():
    x = np.ascontiguousarray(gen()).reshape(-1)
    for eb in (1e-2, 1e-3, 1e-4):
        for b in (8, 16, 32, 64, 128, 256):
            s = oracle.compress(x, eb, oracle.REL, b)
            y = oracle.decompress(s)
            q = oracle.quality(x, y)
            ov = oracle.shift_overhead(s, x)
            print(json.dumps(dict(field=name, n=int(x.size), dtype=str(x.dtype), eb_rel=eb, block=b,
                                  cr=x.nbytes / s.size, psnr=q["psnr"], max_abs_err=q["max_abs_err"],
                                  eb_abs=oracle.read_header(s)["eb_abs"], bits_C=ov["bits_C"],
                                  bits_B=ov["bits_B"], shift_overhead=ov["overhead"])), flush=True)
