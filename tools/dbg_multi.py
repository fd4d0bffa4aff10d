"""Debug: loopback multi fill, report where results differ from the oracle (development tool)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle  # noqa: E402
from paper_conf_ipps_kumark15_b200 import inputs  # noqa: E402
from test_gpu_multi import run_loopback  # noqa: E402

for (m, n, P, nf, kern) in [(2100, 4001, 2, 1, None), (2100, 4001, 2, 4, None), (2100, 4001, 2, 1, "adiag"),
                            (2100, 4001, 1, 1, None), (2100, 2000, 1, 1, None), (768, 4001, 2, 1, None)]:
    probs = [inputs.gen_strings(100 * k + m + n + P, m, n) for k in range(nf)]
    res = run_loopback("lcs", probs, P, kernel=kern)
    for k, ((s, lr, lc), (a, b)) in enumerate(zip(res, probs)):
        ref = oracle.lcs(a, b)
        bad_r = np.nonzero(lr != ref.last_row)[0]
        bad_c = np.nonzero(lc != ref.last_col)[0]
        print(m, n, P, nf, kern, "fill", k, "score", s, ref.score, "bad last_row", len(bad_r),
              bad_r[:5].tolist(), "bad last_col", len(bad_c), bad_c[:5].tolist(),
              (lc[bad_c[:3]].tolist(), ref.last_col[bad_c[:3]].tolist()) if len(bad_c) else "", flush=True)
