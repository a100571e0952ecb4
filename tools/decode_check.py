"""Decode sweep + round-trip check of the EF decoder on a workload's index
(GPU): every list decoded through griffin_debug_decode_list must equal the
corpus, and the decode-only sweep's XOR checksum must equal the XOR of all
docIDs.  Prints one JSON line per block size."""
import json
import sys
import time

import numpy as np

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from synth import make_workload  # noqa: E402

cfg_name = sys.argv[1] if len(sys.argv) > 1 else "c2"
blocks = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [128]
t0 = time.time()
c, ql, cfg = make_workload(cfg_name)
gen_s = time.time() - t0
xor_all = int(np.bitwise_xor.reduce(np.asarray(c.docids))) if c.num_postings else 0
peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if __import__("os").path.exists("MEASURED_PEAKS.json") else 6459.0
for B in blocks:
    ix = g.GriffinIndex(c, block_size=B)
    rng = np.random.default_rng(1)
    terms = list(range(min(50, c.num_terms))) + rng.integers(0, c.num_terms, 200).tolist()
    bad = [t for t in terms if not np.array_equal(ix.griffin_debug_decode_list(t), c.list(t))]
    sw = ix.griffin_debug_decode_all(iters=5)
    gbs = sw["bytes"] / (sw["ms"] / 1e3) / 1e9
    print(json.dumps({"config": cfg_name, "B": B, "gen_s": round(gen_s, 1), "roundtrip_bad": bad[:10],
                      "checksum_ok": (sw["checksum"] & 0xFFFFFFFF) == xor_all, "ms": sw["ms"],
                      "postings": sw["postings"], "bytes": sw["bytes"],
                      "gpostings_s": sw["postings"] / (sw["ms"] / 1e3) / 1e9, "gbs": gbs,
                      "frac": gbs / peak}), flush=True)
    ix.close()
