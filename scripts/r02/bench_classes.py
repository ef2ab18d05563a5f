"""Run bench.py for the given workloads and print one line per kernel class:
{"workload": "<wl>:<class>", "us": per-launch us (graph-profiled)} + the step time."""
import json, subprocess, sys, os
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
for w in sys.argv[1:] or ["c2"]:
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "10", "--warmup", "3",
                          "--workload", w, "--no-cpu-baseline"], capture_output=True, text=True, cwd=os.getcwd())
    line = [l for l in out.stdout.splitlines() if l.startswith("{")]
    if not line:
        print(json.dumps({"workload": w, "error": out.stderr[-500:]})); continue
    d = json.loads(line[-1])
    print(json.dumps({"workload": f"{w}:step_ms", "us": d["ms_per_step"] * 1e3}), flush=True)
    for c, v in d["roofline"]["classes"].items():
        print(json.dumps({"workload": f"{w}:{c}", "us": v["us_per_launch"], "iso_us": v.get("isolated", {}).get("us_per_launch")}), flush=True)
