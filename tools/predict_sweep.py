"""Sweep predict configurations on the DSE workload (not part of the library)."""
import os, subprocess, sys, json
for cfg in (9, 8):
    env = dict(os.environ, DT_PREDICT_CFG=str(cfg))
    out = subprocess.run([sys.executable, "bench.py", "--steps", "3", "--warmup", "3", "--no-cpu", "--e2e-steps", "1"],
                         env=env, capture_output=True, text=True).stdout
    d = json.loads(out.strip().splitlines()[-1])["dse"]
    print(cfg, round(d["predictions_per_s"] / 1e9, 2), "G/s", round(d["roofline"]["frac"], 3), round(d["ms_per_pass"], 2), "ms")
