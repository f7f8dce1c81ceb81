"""Run bench.py over a list of settings and print one summary line each (experiments)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(args, env=None, label=""):
    e = dict(os.environ)
    e.update(env or {})
    p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--no-cpu", "--no-e2e", "--no-side", *args],
                       capture_output=True, text=True, env=e, timeout=600)
    lines = [l for l in p.stdout.splitlines() if l.startswith("{")]
    if not lines:
        print(label, "FAILED", p.stderr[-800:], flush=True)
        return None
    d = json.loads(lines[-1])
    cub = d.get("cublas") or {}
    print(f"{label:40s} {d['config']['workload']:22s} {d['value']:8.1f} TF  cublas {cub.get('value', 0):8.1f}  "
          f"med {d['step_ms']['median']:.4f} ms  kern {d['config']['kernel']['last_kernel']}/{d['config']['kernel']['block_n']}"
          f"  clk {d['clocks']['sm_mhz']} kern-clk {d['clocks'].get('sm_mhz_in_kernel_median', 0):.0f} {d['clocks']['reasons']}", flush=True)
    return d


if __name__ == "__main__":
    spec = json.loads(sys.argv[1])
    for item in spec:
        run(item.get("args", []), item.get("env"), item.get("label", ""))
