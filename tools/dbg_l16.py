"""Debug: one lcs16 fill vs the oracle, print mismatch details (development tool)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle  # noqa: E402
from gpu_util import run_gpu  # noqa: E402
from paper_conf_ipps_kumark15_b200 import inputs  # noqa: E402

for P, E, m, n, seed in [(3, 3, 14000, 15001, 33), (3, 3, 14000, 15001, 34), (3, 2, 14000, 15001, 33),
                         (6, 2, 14000, 15001, 33), (3, 3, 4000, 15001, 33)]:
    os.environ["LDDP_L16_P"], os.environ["LDDP_L16_E"] = str(P), str(E)
    a, b = inputs.gen_strings(seed, m, n)
    got = run_gpu("lcs", "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"))
    ref = oracle.lcs(a, b)
    bc = np.nonzero(got["last_col"] != ref.last_col)[0]
    br = np.nonzero(got["last_row"] != ref.last_row)[0]
    info = got["plan"]
    print(P, E, m, n, seed, "score", got["score"], ref.score, "bad cols", len(bc), bc[:3].tolist(), bc[-3:].tolist(),
          "got", got["last_col"][bc[:3]].tolist(), "ref", ref.last_col[bc[:3]].tolist(), "bad row", len(br), flush=True)
