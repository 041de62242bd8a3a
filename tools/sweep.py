"""Env-knob sweep of one config (dev tool): prints the steady aggregate time per setting."""
import itertools, os, subprocess, sys, json
cfg = sys.argv[1]
grid = json.loads(sys.argv[2])  # {"ENV": [values...]}
rows = sys.argv[3] if len(sys.argv) > 3 else ""
keys = list(grid)
for combo in itertools.product(*[grid[k] for k in keys]):
    env = dict(os.environ, ITERS="4", **{k: str(v) for k, v in zip(keys, combo)})
    out = subprocess.run([sys.executable, "tools/phase_probe.py", cfg] + ([rows] if rows else []), env=env,
                         capture_output=True, text=True).stdout.strip().splitlines()
    last = [l for l in out if l.startswith("wall")][-1:] or ["FAILED " + " ".join(out[-2:])]
    print(dict(zip(keys, combo)), last[0], flush=True)
