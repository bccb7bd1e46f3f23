"""Budget sweep of the AlphaFold-shaped trace with emulated compute (survey §8(d) M2): exposed
transfer time per step vs device budget; B*0 = smallest budget with exposed <= 5% of compute."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
budgets = [float(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "1,2,4,8,16,32").split(",")]
rows = []
for b in budgets:
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--config", "af", "--budget-gib", str(b),
                        "--steps", os.environ.get("SWEEP_STEPS", "4"), "--warmup", "2", "--no-cpu-baseline", "--no-faults",
                        "--policy", os.environ.get("SWEEP_POLICY", "1")], capture_output=True, text=True)
    try:
        d = json.loads(r.stdout.strip().splitlines()[-1])
    except Exception:
        print("budget", b, "failed:", r.stderr[-600:], flush=True)
        continue
    ce = d.get("compute_emulation") or {}
    row = {"budget_gib": b, "ms_per_step": d["ms_per_step"], "compute_ms": ce.get("compute_ms_per_step"),
           "exposed_ms": ce.get("exposed_ms_per_step"), "exposed_frac": ce.get("exposed_frac_of_compute"),
           "compute_only_ms": ce.get("compute_only_ms_per_step"), "exposed_vs_compute_only_ms": ce.get("exposed_vs_compute_only_ms"),
           "exposed_vs_compute_only_frac": ce.get("exposed_vs_compute_only_frac"),
           "migration_gbs": d["value"], "h2d_GB_step": round(d["h2d_bytes_per_step"] / 1e9, 3),
           "d2h_GB_step": round(d["d2h_bytes_per_step"] / 1e9, 3), "plan_us": d["plan_us"],
           "h2d_dma_gbs": d["pcie"]["h2d_dma_gbs"], "d2h_dma_gbs": d["pcie"]["d2h_dma_gbs"]}
    rows.append(row)
    print(json.dumps(row), flush=True)
ok = [r for r in rows if r["exposed_frac"] is not None and r["exposed_frac"] <= 0.05]
ok2 = [r for r in rows if r.get("exposed_vs_compute_only_frac") is not None and r["exposed_vs_compute_only_frac"] <= 0.05]
print(json.dumps({"policy": int(os.environ.get("SWEEP_POLICY", "1")),
                  "B_star_0_gib": min(r["budget_gib"] for r in ok) if ok else None,
                  "B_star_0_gib_vs_compute_only": min(r["budget_gib"] for r in ok2) if ok2 else None, "rows": rows}))
