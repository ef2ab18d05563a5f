"""bench.py for the given workloads: device value and the C-ABI host-buffer e2e value."""
import json, subprocess, sys, os
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
for w in sys.argv[1:] or ["c2"]:
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "20", "--warmup", "3",
                          "--workload", w, "--no-cpu-baseline"], capture_output=True, text=True, cwd=os.getcwd())
    line = [l for l in out.stdout.splitlines() if l.startswith("{")]
    if not line:
        print(json.dumps({"workload": w, "error": out.stderr[-400:]})); continue
    d = json.loads(line[-1])
    print(json.dumps({"workload": w, "value": d["value"], "e2e": d["e2e"]["value"], "ms": d["ms_per_step"]}), flush=True)
