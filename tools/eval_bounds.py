"""Held-out evaluation of the reuse-bound choices: modelled plan time
of fixed (0,0,0), the whole-plan sweep, the per-vector sweep and the per-vector regression on
the configs tools/train_bounds.py held out.  Writes profiles/bounds_eval_r01.json."""
import json
import sys
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
sys.path.insert(0, str(ROOT / "tools"))
import paper_conf_ipps_wangr0e22_b200 as M  # noqa: E402
from train_bounds import context, heldout, workload  # noqa: E402

rows = []
for c in heldout():
    wl = workload(c)
    ctx = context(c, wl)
    n = c["n_gpus"]
    p = {m: M.micco_plan_stages(ctx.h, n, *a)[2] for m, a in
         {"fixed000": ("fixed", [0, 0, 0]), "sweep": ("fixed", None), "stage_sweep": ("stage_sweep",),
          "regression": ("regression",)}.items()}
    ctx.close()
    rows.append(dict(config=c, **p))
keys = ["sweep", "stage_sweep", "regression"]
summary = {k: {"mean_ratio_vs_fixed000": float(np.mean([r[k] / r["fixed000"] for r in rows])),
               "best_or_tied_share": float(np.mean([r[k] <= min(r[j] for j in keys) * (1 + 1e-9) for r in rows]))}
           for k in keys}
out = {"n_heldout": len(rows), "summary": summary, "rows": rows}
(ROOT / "profiles" / "bounds_eval_r01.json").write_text(json.dumps(out, indent=1))
print(json.dumps(summary, indent=1))
